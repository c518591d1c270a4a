// gat.cu -- a6 / a9: fused GAT layer (Fig. 2 L95-L123, Fig. 3 L159 src lines 9-23).
//
// Forward: the paper's FSM splits the GAT forward into 2 fused units at the Div (L391-L393:
// AggSum of exp, then Div -> Mul -> AggSum).  On B200 it is ONE pass over in(v): an online
// softmax keeps (running max m, running sum S, running weighted row acc) in registers, so no
// E-sized intermediate and no second gather of T are needed.  lse = m + log S is saved for the
// backward.
//
// Backward (§6.3.4: the Aggregation stage becomes the Source stage on the reverse CSR):
//   row pass (gat_bwd_prep): dA = dY act'(Y), c[v,h] = <dA[v,h], A[v,h]> (= sum_e a_e <dA_v, T_u>,
//     which removes the softmax-Jacobian pass), packed with er and lse into one record D[v];
//   source-major pass (gat_bwd, REV CSR): per u, per out-edge (u->v): a_e = exp(LReLU(s_e) - lse_v),
//     g_e = <dA_v, T_u>, ds_e = a_e (g_e - c_v) LReLU'(s_e); dT_u += a_e dA_v, del_u += ds_e in
//     registers (no atomics);
//   destination-major pass (gat_der, FWD CSR): der_v = sum_{e in in(v)} ds_e, recomputing ds_e from
//     the L2-resident T / el tables instead of materialising an E x H array.
//
// Two lane mappings:
//   * head-per-lane ("hpl", H | 32, F % 4 == 0, F <= 32): lane = (edge slot, head), each lane owns a
//     whole head row of F floats: one exp per (edge, head), dot products stay inside a lane;
//   * chunked (any H, F): a row is split into float4 (or float) chunks over L lanes per edge,
//     head dot products by a segmented shuffle reduction.
#include <math.h>

#include "common.cuh"

#ifndef GAT_MB_FWD
#define GAT_MB_FWD 3   // min resident 256-thread blocks per SM (<= 85 regs): measured best on Reddit
#endif
#ifndef GAT_MB_BWD
#define GAT_MB_BWD 3
#endif

namespace seastar {

__device__ __forceinline__ float lrelu(float x, float slope) { return x > 0.f ? x : slope * x; }

struct GatFwdArgs {
    const int32_t* perm; const int32_t* off; const int32_t* nbr;
    int64_t row_begin, row_end, vbase;
    const float* T; const float* el; const float* er;
    int H, F; int64_t ld; float slope;
    const float* bias; int act;
    float* A; float* Y; float* lse;
    float* B; float* bsum;   // optional: der factors (see k_gat_fwd_hpl)
};

// lane geometry of the chunked kernels: chunk `chunk` covers floats [chunk*VEC, chunk*VEC+VEC)
// of a row of W = H*F floats; with VEC = 4 every chunk lies inside one head (F % 4 == 0 or H == 1)
template <int VEC>
__device__ __forceinline__ int head_of(int chunk, int F, int H) {
    return H == 1 ? 0 : (chunk * VEC) / F;
}

// ============================================================================================
// forward
// ============================================================================================
template <int VEC, int L, int RL>
__global__ void __launch_bounds__(256) k_gat_fwd(const GatFwdArgs a) {
    constexpr int S = RL / L;
    constexpr int UB = (L < 4 ? L : 4);
    const int lane = threadIdx.x & 31;
    const int gl = lane % RL;
    const int slot = gl / L;
    const int c = gl % L;
    const unsigned gmask = (RL == 32) ? 0xffffffffu : (((1u << RL) - 1u) << ((lane / RL) * RL));
    const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t row = a.row_begin + warp * (32 / RL) + lane / RL;
    const bool valid = row < a.row_end;
    const int beg = valid ? __ldg(a.off + row) : 0;
    const int end = valid ? __ldg(a.off + row + 1) : 0;
    const int64_t v = valid ? (int64_t)__ldg(a.perm + row) - a.vbase : 0;
    const int W = a.H * a.F;
    const int C = (W + VEC - 1) / VEC;
    const int chunk = c;                       // C <= L (checked on the host)
    const bool active = chunk < C;
    const int h = active ? head_of<VEC>(chunk, a.F, a.H) : 0;
    const int64_t col = (int64_t)chunk * VEC;
    const float erv = (valid && active) ? __ldg(a.er + v * a.H + h) : 0.f;

    const bool SB = a.B != nullptr;     // fallback path: runtime flag
    float m = -INFINITY, ssum = 0.f, acc[VEC], pacc[VEC], psum = 0.f;
#pragma unroll
    for (int i = 0; i < VEC; ++i) acc[i] = pacc[i] = 0.f;

    int nxt = (gl < end - beg) ? __ldcs(a.nbr + beg + gl) : 0;   // index prefetch (gcn.cu)
    for (int base = beg; base < end; base += RL) {
        const int n = min(RL, end - base);
        const int my = nxt;
        nxt = (gl < end - base - RL) ? __ldcs(a.nbr + base + RL + gl) : 0;
#pragma unroll
        for (int j0 = 0; j0 < L; j0 += UB) {
            if (j0 * S >= n) break;
            float z[UB], val[UB][VEC];
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) {
                const int k = (j0 + jj) * S + slot;
                const int u = __shfl_sync(gmask, my, k & (RL - 1), RL);
                if (k < n && active) {
                    z[jj] = lrelu(__ldg(a.el + (int64_t)u * a.H + h) + erv, a.slope);
                    load_vec<VEC>(a.T + (int64_t)u * a.ld + col, val[jj]);
                } else {
                    z[jj] = -INFINITY;
#pragma unroll
                    for (int i = 0; i < VEC; ++i) val[jj][i] = 0.f;
                }
            }
            float mb = m;
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) mb = fmaxf(mb, z[jj]);
            const float corr = (m == -INFINITY) ? 0.f : expf(m - mb);
            ssum *= corr;
            psum *= corr;
#pragma unroll
            for (int i = 0; i < VEC; ++i) { acc[i] *= corr; pacc[i] *= corr; }
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) {
                const float p = (z[jj] == -INFINITY) ? 0.f : expf(z[jj] - mb);
                ssum += p;
                const float pp = (SB && z[jj] > 0.f) ? p : 0.f;
                psum += pp;
#pragma unroll
                for (int i = 0; i < VEC; ++i) {
                    acc[i] = fmaf(p, val[jj][i], acc[i]);
                    pacc[i] = fmaf(pp, val[jj][i], pacc[i]);
                }
            }
            m = mb;
        }
    }
    // merge the edge slots: online-softmax combine, fixed tree
#pragma unroll
    for (int o = L; o < RL; o <<= 1) {
        const float mo = __shfl_xor_sync(gmask, m, o, RL);
        const float so = __shfl_xor_sync(gmask, ssum, o, RL);
        float ao[VEC];
#pragma unroll
        for (int i = 0; i < VEC; ++i) ao[i] = __shfl_xor_sync(gmask, acc[i], o, RL);
        const float mn = fmaxf(m, mo);
        const float ca = (m == -INFINITY) ? 0.f : expf(m - mn);
        const float cb = (mo == -INFINITY) ? 0.f : expf(mo - mn);
        ssum = ssum * ca + so * cb;
        psum = psum * ca + __shfl_xor_sync(gmask, psum, o, RL) * cb;
#pragma unroll
        for (int i = 0; i < VEC; ++i) {
            acc[i] = acc[i] * ca + ao[i] * cb;
            pacc[i] = pacc[i] * ca + __shfl_xor_sync(gmask, pacc[i], o, RL) * cb;
        }
        m = mn;
    }
    if (!valid || slot != 0 || !active) return;
    const float inv = ssum > 0.f ? 1.f / ssum : 0.f;
    float outA[VEC], outY[VEC];
#pragma unroll
    for (int i = 0; i < VEC; ++i) {
        const float av = acc[i] * inv;
        outA[i] = av;
        const int64_t cc = col + i;
        outY[i] = act_apply(a.act, av + ((a.bias && cc < W) ? __ldg(a.bias + cc) : 0.f));
    }
    float* pa = a.A + v * a.ld + col;
    float* py = a.Y + v * a.ld + col;
    if (col + VEC <= W) {
        store_vec<VEC>(pa, outA);
        store_vec<VEC>(py, outY);
    } else {
        for (int i = 0; i < VEC && col + i < W; ++i) { pa[i] = outA[i]; py[i] = outY[i]; }
    }
    if (SB) {
        float* pb = a.B + v * a.ld + col;
        for (int i = 0; i < VEC && col + i < W; ++i) pb[i] = a.slope * outA[i] + (1.f - a.slope) * pacc[i] * inv;
    }
    if ((a.H == 1 && chunk == 0) || (a.H > 1 && col % a.F == 0)) {
        a.lse[v * a.H + h] = ssum > 0.f ? m + logf(ssum) : -INFINITY;
        if (SB) a.bsum[v * a.H + h] = ssum > 0.f ? a.slope + (1.f - a.slope) * psum * inv : 0.f;
    }
}

// head-per-lane forward: warp per destination row; lane = (slot, head), S = 32/H edge slots.
// SB: also accumulate the positive-logit part P_v = sum_{e: s_e > 0} a_e T_u (same gathered rows), from
// which the epilogue writes B_v = sum_e a_e LReLU'(s_e) T_u and b_v = sum_e a_e LReLU'(s_e) -- the two
// forward-only factors of der_v = <dA_v, B_v> - c_v b_v (so the backward needs no dst-major pass).
template <int F4, bool SB>
__global__ void __launch_bounds__(256, GAT_MB_FWD) k_gat_fwd_hpl(const GatFwdArgs a) {
    constexpr int F = 4 * F4;
    constexpr int UB = F4 <= 2 ? 4 : (F4 <= 4 ? 2 : 1);
    const int H = a.H;
    const int S = 32 / H;
    const int lane = threadIdx.x & 31;
    const int h = lane % H, slot = lane / H;
    const int64_t row = a.row_begin + ((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5);
    if (row >= a.row_end) return;                      // warp-uniform
    const int beg = __ldg(a.off + row), end = __ldg(a.off + row + 1);
    const int64_t v = (int64_t)__ldg(a.perm + row) - a.vbase;
    const float erv = __ldg(a.er + v * H + h);
    const int64_t hoff = (int64_t)h * F;
    float m = -INFINITY, ssum = 0.f, acc[F], pacc[SB ? F : 1], psum = 0.f;
#pragma unroll
    for (int i = 0; i < F; ++i) acc[i] = 0.f;
#pragma unroll
    for (int i = 0; i < (SB ? F : 1); ++i) pacc[i] = 0.f;
    int nxt = (lane < end - beg) ? __ldcs(a.nbr + beg + lane) : 0;   // index prefetch (gcn.cu)
    for (int base = beg; base < end; base += 32) {
        const int n = min(32, end - base);
        const int my = nxt;
        nxt = (lane < end - base - 32) ? __ldcs(a.nbr + base + 32 + lane) : 0;
        for (int i0 = 0; i0 < H; i0 += UB) {             // this slot's edges: k = slot + S * i
            if (i0 * S >= n) break;
            float z[UB], x[UB][F];
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) {
                const int k = slot + S * (i0 + jj);
                const int u = __shfl_sync(0xffffffffu, my, k & 31);
                if (k < n && i0 + jj < H) {
                    z[jj] = lrelu(__ldg(a.el + (int64_t)u * H + h) + erv, a.slope);
                    const float* tp = a.T + (int64_t)u * a.ld + hoff;
#pragma unroll
                    for (int q = 0; q < F4; ++q) {
                        const float4 t4 = ldg4(tp + 4 * q);
                        x[jj][4 * q] = t4.x; x[jj][4 * q + 1] = t4.y; x[jj][4 * q + 2] = t4.z; x[jj][4 * q + 3] = t4.w;
                    }
                } else {
                    z[jj] = -INFINITY;
#pragma unroll
                    for (int i = 0; i < F; ++i) x[jj][i] = 0.f;
                }
            }
            float mb = m;
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) mb = fmaxf(mb, z[jj]);
            if (mb > m) {                                 // rescale only when the running max moves
                const float corr = (m == -INFINITY) ? 0.f : expf(m - mb);
                ssum *= corr;
#pragma unroll
                for (int i = 0; i < F; ++i) acc[i] *= corr;
                if (SB) {
                    psum *= corr;
#pragma unroll
                    for (int i = 0; i < (SB ? F : 1); ++i) pacc[i] *= corr;
                }
                m = mb;
            }
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) {
                const float p = (z[jj] == -INFINITY) ? 0.f : expf(z[jj] - m);
                ssum += p;
#pragma unroll
                for (int i = 0; i < F; ++i) acc[i] = fmaf(p, x[jj][i], acc[i]);
                if (SB) {
                    const float pp = z[jj] > 0.f ? p : 0.f;
                    psum += pp;
#pragma unroll
                    for (int i = 0; i < (SB ? F : 1); ++i) pacc[i] = fmaf(pp, x[jj][i], pacc[i]);
                }
            }
        }
    }
    for (int o = H; o < 32; o <<= 1) {
        const float mo = __shfl_xor_sync(0xffffffffu, m, o);
        const float so = __shfl_xor_sync(0xffffffffu, ssum, o);
        const float mn = fmaxf(m, mo);
        const float ca = (m == -INFINITY) ? 0.f : expf(m - mn);
        const float cb = (mo == -INFINITY) ? 0.f : expf(mo - mn);
        ssum = ssum * ca + so * cb;
#pragma unroll
        for (int i = 0; i < F; ++i) acc[i] = acc[i] * ca + __shfl_xor_sync(0xffffffffu, acc[i], o) * cb;
        if (SB) {
            psum = psum * ca + __shfl_xor_sync(0xffffffffu, psum, o) * cb;
#pragma unroll
            for (int i = 0; i < (SB ? F : 1); ++i) pacc[i] = pacc[i] * ca + __shfl_xor_sync(0xffffffffu, pacc[i], o) * cb;
        }
        m = mn;
    }
    if (slot != 0) return;
    const float inv = ssum > 0.f ? 1.f / ssum : 0.f;
    float* pa = a.A + v * a.ld + hoff;
    float* py = a.Y + v * a.ld + hoff;
#pragma unroll
    for (int q = 0; q < F4; ++q) {
        float o4[4], y4[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            o4[i] = acc[4 * q + i] * inv;
            y4[i] = act_apply(a.act, o4[i] + (a.bias ? __ldg(a.bias + hoff + 4 * q + i) : 0.f));
        }
        *reinterpret_cast<float4*>(pa + 4 * q) = make_float4(o4[0], o4[1], o4[2], o4[3]);
        *reinterpret_cast<float4*>(py + 4 * q) = make_float4(y4[0], y4[1], y4[2], y4[3]);
        if (SB) {
            float b4[4];
#pragma unroll
            for (int i = 0; i < 4; ++i) b4[i] = a.slope * o4[i] + (1.f - a.slope) * pacc[(4 * q + i) % (SB ? F : 1)] * inv;
            *reinterpret_cast<float4*>(a.B + v * a.ld + hoff + 4 * q) = make_float4(b4[0], b4[1], b4[2], b4[3]);
        }
    }
    a.lse[v * H + h] = ssum > 0.f ? m + logf(ssum) : -INFINITY;
    if (SB) a.bsum[v * H + h] = ssum > 0.f ? a.slope + (1.f - a.slope) * psum * inv : 0.f;
}

// ============================================================================================
// backward
// ============================================================================================
struct GatBwdArgs {
    const int32_t* perm; const int32_t* off; const int32_t* nbr;
    int64_t row_begin, row_end, vbase;
    const float* T;      // gathered (der) or owned (src-major) rows
    const float* el;     // gathered (der) or owned (src-major)
    const float* D;      // packed records: gathered (src-major) or owned (der)
    int H, F; int64_t ldt, ldd; float slope;
    float* dT; float* del;   // src-major outputs
    float* der;              // der output
};

__device__ __forceinline__ int rec_aux_offset(int W) { return (W + 3) & ~3; }

// chunked source-major backward (REV CSR): dT_u, del_u
template <int VEC, int L, int RL>
__global__ void __launch_bounds__(256) k_gat_bwd(const GatBwdArgs a) {
    constexpr int S = RL / L;
    constexpr int UB = (L < 4 ? L : 4);
    const int lane = threadIdx.x & 31;
    const int gl = lane % RL;
    const int slot = gl / L;
    const int c = gl % L;
    const unsigned gmask = (RL == 32) ? 0xffffffffu : (((1u << RL) - 1u) << ((lane / RL) * RL));
    const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t row = a.row_begin + warp * (32 / RL) + lane / RL;
    const bool valid = row < a.row_end;
    const int beg = valid ? __ldg(a.off + row) : 0;
    const int end = valid ? __ldg(a.off + row + 1) : 0;
    const int64_t u = valid ? (int64_t)__ldg(a.perm + row) - a.vbase : 0;
    const int W = a.H * a.F;
    const int C = (W + VEC - 1) / VEC;
    const int chunk = c;
    const bool active = chunk < C;
    const int h = active ? head_of<VEC>(chunk, a.F, a.H) : (a.H - 1);
    const int64_t col = (int64_t)chunk * VEC;
    const int lph = (a.H == 1) ? C : (a.F / VEC);      // lanes of head h inside the edge group
    const int hc = active ? (a.H == 1 ? chunk : chunk - h * lph) : 0;
    const int hs = c - hc;
    const int aux0 = rec_aux_offset(W);

    float t[VEC];
    if (valid && active) load_vec<VEC>(a.T + u * a.ldt + col, t);
#pragma unroll
    for (int i = 0; i < VEC; ++i)   // padding columns never enter the head dot products
        if (!(valid && active) || col + i >= W) t[i] = 0.f;
    const float elu = (valid && active) ? __ldg(a.el + u * a.H + h) : 0.f;
    float acc[VEC], dl = 0.f;
#pragma unroll
    for (int i = 0; i < VEC; ++i) acc[i] = 0.f;

    int nxt = (gl < end - beg) ? __ldcs(a.nbr + beg + gl) : 0;   // index prefetch (gcn.cu)
    for (int base = beg; base < end; base += RL) {
        const int n = min(RL, end - base);
        const int myv = nxt;
        nxt = (gl < end - base - RL) ? __ldcs(a.nbr + base + RL + gl) : 0;
#pragma unroll
        for (int j0 = 0; j0 < L; j0 += UB) {
            if (j0 * S >= n) break;
            float dA[UB][VEC], er[UB], lse[UB], cv[UB];
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) {
                const int k = (j0 + jj) * S + slot;
                const int v = __shfl_sync(gmask, myv, k & (RL - 1), RL);
                if (k < n && active) {
                    const float* rec = a.D + (int64_t)v * a.ldd;
                    load_vec<VEC>(rec + col, dA[jj]);
#pragma unroll
                    for (int i = 0; i < VEC; ++i)
                        if (col + i >= W) dA[jj][i] = 0.f;
                    const float* aux = rec + aux0 + 4 * h;
                    er[jj] = __ldg(aux); lse[jj] = __ldg(aux + 1); cv[jj] = __ldg(aux + 2);
                } else {
#pragma unroll
                    for (int i = 0; i < VEC; ++i) dA[jj][i] = 0.f;
                    er[jj] = 0.f; lse[jj] = INFINITY; cv[jj] = 0.f;
                }
            }
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) {
                const int k = (j0 + jj) * S + slot;
                float gp = 0.f;
#pragma unroll
                for (int i = 0; i < VEC; ++i) gp = fmaf(dA[jj][i], t[i], gp);
#pragma unroll
                for (int o = 1; o < L; o <<= 1) {
                    const float x = __shfl_down_sync(gmask, gp, o, L);
                    if (hc + o < lph) gp += x;
                }
                const float g = __shfl_sync(gmask, gp, hs, L);
                if (k < n && active) {
                    const float s = elu + er[jj];
                    const float al = expf(lrelu(s, a.slope) - lse[jj]);
                    dl += al * (g - cv[jj]) * (s > 0.f ? 1.f : a.slope);
#pragma unroll
                    for (int i = 0; i < VEC; ++i) acc[i] = fmaf(al, dA[jj][i], acc[i]);
                }
            }
        }
    }
#pragma unroll
    for (int o = L; o < RL; o <<= 1) {
#pragma unroll
        for (int i = 0; i < VEC; ++i) acc[i] += __shfl_xor_sync(gmask, acc[i], o, RL);
        dl += __shfl_xor_sync(gmask, dl, o, RL);
    }
    if (!valid || slot != 0 || !active) return;
    float* pd = a.dT + u * a.ldt + col;
    if (col + VEC <= W) store_vec<VEC>(pd, acc);
    else
        for (int i = 0; i < VEC && col + i < W; ++i) pd[i] = acc[i];
    if (hc == 0) a.del[u * a.H + h] = dl;
}

// chunked destination-major der pass (FWD CSR): der_v = sum_{e in in(v)} ds_e
template <int VEC, int L, int RL>
__global__ void __launch_bounds__(256) k_gat_der(const GatBwdArgs a) {
    constexpr int S = RL / L;
    constexpr int UB = (L < 4 ? L : 4);
    const int lane = threadIdx.x & 31;
    const int gl = lane % RL;
    const int slot = gl / L;
    const int c = gl % L;
    const unsigned gmask = (RL == 32) ? 0xffffffffu : (((1u << RL) - 1u) << ((lane / RL) * RL));
    const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t row = a.row_begin + warp * (32 / RL) + lane / RL;
    const bool valid = row < a.row_end;
    const int beg = valid ? __ldg(a.off + row) : 0;
    const int end = valid ? __ldg(a.off + row + 1) : 0;
    const int64_t v = valid ? (int64_t)__ldg(a.perm + row) - a.vbase : 0;
    const int W = a.H * a.F;
    const int C = (W + VEC - 1) / VEC;
    const int chunk = c;
    const bool active = chunk < C;
    const int h = active ? head_of<VEC>(chunk, a.F, a.H) : (a.H - 1);
    const int64_t col = (int64_t)chunk * VEC;
    const int lph = (a.H == 1) ? C : (a.F / VEC);
    const int hc = active ? (a.H == 1 ? chunk : chunk - h * lph) : 0;
    const int hs = c - hc;

    float d[VEC];
    float erv = 0.f, lsev = 0.f, cvv = 0.f;
    if (valid && active) {
        const float* rec = a.D + v * a.ldd;
        load_vec<VEC>(rec + col, d);
        const float* aux = rec + rec_aux_offset(W) + 4 * h;
        erv = __ldg(aux); lsev = __ldg(aux + 1); cvv = __ldg(aux + 2);
    }
#pragma unroll
    for (int i = 0; i < VEC; ++i)
        if (!(valid && active) || col + i >= W) d[i] = 0.f;
    float dr = 0.f;
    int nxt = (gl < end - beg) ? __ldcs(a.nbr + beg + gl) : 0;   // index prefetch (gcn.cu)
    for (int base = beg; base < end; base += RL) {
        const int n = min(RL, end - base);
        const int my = nxt;
        nxt = (gl < end - base - RL) ? __ldcs(a.nbr + base + RL + gl) : 0;
#pragma unroll
        for (int j0 = 0; j0 < L; j0 += UB) {
            if (j0 * S >= n) break;
            float t[UB][VEC], elu[UB];
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) {
                const int k = (j0 + jj) * S + slot;
                const int u = __shfl_sync(gmask, my, k & (RL - 1), RL);
                if (k < n && active) {
                    load_vec<VEC>(a.T + (int64_t)u * a.ldt + col, t[jj]);
#pragma unroll
                    for (int i = 0; i < VEC; ++i)
                        if (col + i >= W) t[jj][i] = 0.f;
                    elu[jj] = __ldg(a.el + (int64_t)u * a.H + h);
                } else {
#pragma unroll
                    for (int i = 0; i < VEC; ++i) t[jj][i] = 0.f;
                    elu[jj] = 0.f;
                }
            }
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) {
                const int k = (j0 + jj) * S + slot;
                float gp = 0.f;
#pragma unroll
                for (int i = 0; i < VEC; ++i) gp = fmaf(d[i], t[jj][i], gp);
#pragma unroll
                for (int o = 1; o < L; o <<= 1) {
                    const float x = __shfl_down_sync(gmask, gp, o, L);
                    if (hc + o < lph) gp += x;
                }
                const float g = __shfl_sync(gmask, gp, hs, L);
                if (k < n && active) {
                    const float s = elu[jj] + erv;
                    const float al = expf(lrelu(s, a.slope) - lsev);
                    dr += al * (g - cvv) * (s > 0.f ? 1.f : a.slope);
                }
            }
        }
    }
#pragma unroll
    for (int o = L; o < RL; o <<= 1) dr += __shfl_xor_sync(gmask, dr, o, RL);
    if (!valid || slot != 0 || !active) return;
    if (hc == 0) a.der[v * a.H + h] = dr;
}

// head-per-lane source-major backward (REV CSR)
template <int F4>
__global__ void __launch_bounds__(256, GAT_MB_BWD) k_gat_bwd_hpl(const GatBwdArgs a) {
    constexpr int F = 4 * F4;
    constexpr int UB = F4 <= 2 ? 4 : (F4 <= 4 ? 2 : 1);
    const int H = a.H, S = 32 / H;
    const int lane = threadIdx.x & 31;
    const int h = lane % H, slot = lane / H;
    const int64_t row = a.row_begin + ((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5);
    if (row >= a.row_end) return;
    const int beg = __ldg(a.off + row), end = __ldg(a.off + row + 1);
    const int64_t u = (int64_t)__ldg(a.perm + row) - a.vbase;
    const int64_t hoff = (int64_t)h * F;
    const int aux0 = rec_aux_offset(H * F) + 4 * h;
    float t[F], acc[F];
#pragma unroll
    for (int q = 0; q < F4; ++q) {
        const float4 t4 = ldg4(a.T + u * a.ldt + hoff + 4 * q);
        t[4 * q] = t4.x; t[4 * q + 1] = t4.y; t[4 * q + 2] = t4.z; t[4 * q + 3] = t4.w;
    }
#pragma unroll
    for (int i = 0; i < F; ++i) acc[i] = 0.f;
    const float elu = __ldg(a.el + u * H + h);
    float dl = 0.f;
    int nxt = (lane < end - beg) ? __ldcs(a.nbr + beg + lane) : 0;   // index prefetch (gcn.cu)
    for (int base = beg; base < end; base += 32) {
        const int n = min(32, end - base);
        const int my = nxt;
        nxt = (lane < end - base - 32) ? __ldcs(a.nbr + base + 32 + lane) : 0;
        for (int i0 = 0; i0 < H; i0 += UB) {
            if (i0 * S >= n) break;
            float d[UB][F], ax[UB][3];
            bool ok[UB];
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) {
                const int k = slot + S * (i0 + jj);
                const int v = __shfl_sync(0xffffffffu, my, k & 31);
                ok[jj] = k < n && i0 + jj < H;
                if (ok[jj]) {
                    const float* rec = a.D + (int64_t)v * a.ldd;
#pragma unroll
                    for (int q = 0; q < F4; ++q) {
                        const float4 d4 = ldg4(rec + hoff + 4 * q);
                        d[jj][4 * q] = d4.x; d[jj][4 * q + 1] = d4.y; d[jj][4 * q + 2] = d4.z; d[jj][4 * q + 3] = d4.w;
                    }
                    const float4 x4 = ldg4(rec + aux0);
                    ax[jj][0] = x4.x; ax[jj][1] = x4.y; ax[jj][2] = x4.z;
                } else {
#pragma unroll
                    for (int i = 0; i < F; ++i) d[jj][i] = 0.f;
                    ax[jj][0] = 0.f; ax[jj][1] = INFINITY; ax[jj][2] = 0.f;
                }
            }
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) {
                if (!ok[jj]) continue;
                float g = 0.f;
#pragma unroll
                for (int i = 0; i < F; ++i) g = fmaf(d[jj][i], t[i], g);
                const float s = elu + ax[jj][0];
                const float al = expf(lrelu(s, a.slope) - ax[jj][1]);
                dl += al * (g - ax[jj][2]) * (s > 0.f ? 1.f : a.slope);
#pragma unroll
                for (int i = 0; i < F; ++i) acc[i] = fmaf(al, d[jj][i], acc[i]);
            }
        }
    }
    for (int o = H; o < 32; o <<= 1) {
#pragma unroll
        for (int i = 0; i < F; ++i) acc[i] += __shfl_xor_sync(0xffffffffu, acc[i], o);
        dl += __shfl_xor_sync(0xffffffffu, dl, o);
    }
    if (slot != 0) return;
    float* pd = a.dT + u * a.ldt + hoff;
#pragma unroll
    for (int q = 0; q < F4; ++q)
        *reinterpret_cast<float4*>(pd + 4 * q) = make_float4(acc[4 * q], acc[4 * q + 1], acc[4 * q + 2], acc[4 * q + 3]);
    a.del[u * H + h] = dl;
}

// head-per-lane destination-major der pass (FWD CSR)
template <int F4>
__global__ void __launch_bounds__(256) k_gat_der_hpl(const GatBwdArgs a) {
    constexpr int F = 4 * F4;
    constexpr int UB = F4 <= 2 ? 4 : (F4 <= 4 ? 2 : 1);
    const int H = a.H, S = 32 / H;
    const int lane = threadIdx.x & 31;
    const int h = lane % H, slot = lane / H;
    const int64_t row = a.row_begin + ((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5);
    if (row >= a.row_end) return;
    const int beg = __ldg(a.off + row), end = __ldg(a.off + row + 1);
    const int64_t v = (int64_t)__ldg(a.perm + row) - a.vbase;
    const int64_t hoff = (int64_t)h * F;
    const float* rec = a.D + v * a.ldd;
    float d[F];
#pragma unroll
    for (int q = 0; q < F4; ++q) {
        const float4 d4 = ldg4(rec + hoff + 4 * q);
        d[4 * q] = d4.x; d[4 * q + 1] = d4.y; d[4 * q + 2] = d4.z; d[4 * q + 3] = d4.w;
    }
    const float4 x4 = ldg4(rec + rec_aux_offset(H * F) + 4 * h);
    const float erv = x4.x, lsev = x4.y, cvv = x4.z;
    float dr = 0.f;
    int nxt = (lane < end - beg) ? __ldcs(a.nbr + beg + lane) : 0;   // index prefetch (gcn.cu)
    for (int base = beg; base < end; base += 32) {
        const int n = min(32, end - base);
        const int my = nxt;
        nxt = (lane < end - base - 32) ? __ldcs(a.nbr + base + 32 + lane) : 0;
        for (int i0 = 0; i0 < H; i0 += UB) {
            if (i0 * S >= n) break;
            float t[UB][F], elu[UB];
            bool ok[UB];
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) {
                const int k = slot + S * (i0 + jj);
                const int u = __shfl_sync(0xffffffffu, my, k & 31);
                ok[jj] = k < n && i0 + jj < H;
                if (ok[jj]) {
                    const float* tp = a.T + (int64_t)u * a.ldt + hoff;
#pragma unroll
                    for (int q = 0; q < F4; ++q) {
                        const float4 t4 = ldg4(tp + 4 * q);
                        t[jj][4 * q] = t4.x; t[jj][4 * q + 1] = t4.y; t[jj][4 * q + 2] = t4.z; t[jj][4 * q + 3] = t4.w;
                    }
                    elu[jj] = __ldg(a.el + (int64_t)u * H + h);
                } else {
#pragma unroll
                    for (int i = 0; i < F; ++i) t[jj][i] = 0.f;
                    elu[jj] = 0.f;
                }
            }
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) {
                if (!ok[jj]) continue;
                float g = 0.f;
#pragma unroll
                for (int i = 0; i < F; ++i) g = fmaf(d[i], t[jj][i], g);
                const float s = elu[jj] + erv;
                const float al = expf(lrelu(s, a.slope) - lsev);
                dr += al * (g - cvv) * (s > 0.f ? 1.f : a.slope);
            }
        }
    }
    for (int o = H; o < 32; o <<= 1) dr += __shfl_xor_sync(0xffffffffu, dr, o);
    if (slot == 0) a.der[v * H + h] = dr;
}

// ============================================================================================
// single-head kernels: each lane owns VPL consecutive float4 chunks of the row, L lanes per edge
// (L <= 4), S = RL / L edge slots; g = <dA, T> by an L-lane xor reduction
// ============================================================================================
template <int VPL>
__device__ __forceinline__ void load_chunks(const float* p, int col0, int W, float (&x)[4 * VPL]) {
#pragma unroll
    for (int q = 0; q < VPL; ++q) {
        const int col = col0 + 4 * q;
        if (col < W) {
            const float4 t = ldg4(p + col);
            x[4 * q] = t.x; x[4 * q + 1] = t.y; x[4 * q + 2] = t.z; x[4 * q + 3] = t.w;
#pragma unroll
            for (int i = 0; i < 4; ++i)
                if (col + i >= W) x[4 * q + i] = 0.f;
        } else {
#pragma unroll
            for (int i = 0; i < 4; ++i) x[4 * q + i] = 0.f;
        }
    }
}

template <int VPL, int L, int RL, bool SB>
__global__ void __launch_bounds__(256, GAT_MB_FWD) k_gat_fwd_h1(const GatFwdArgs a) {
    constexpr int NV = 4 * VPL, S = RL / L, UB = VPL <= 2 ? 4 : 2;
    constexpr int NP = SB ? NV : 1;
    const int lane = threadIdx.x & 31;
    const int gl = lane % RL, slot = gl / L, c = gl % L;
    const unsigned gmask = (RL == 32) ? 0xffffffffu : (((1u << RL) - 1u) << ((lane / RL) * RL));
    const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t row = a.row_begin + warp * (32 / RL) + lane / RL;
    const bool valid = row < a.row_end;
    const int beg = valid ? __ldg(a.off + row) : 0;
    const int end = valid ? __ldg(a.off + row + 1) : 0;
    const int64_t v = valid ? (int64_t)__ldg(a.perm + row) - a.vbase : 0;
    const int W = a.F, col0 = c * NV;
    const float erv = valid ? __ldg(a.er + v) : 0.f;
    float m = -INFINITY, ssum = 0.f, acc[NV], pacc[NP], psum = 0.f;
#pragma unroll
    for (int i = 0; i < NV; ++i) acc[i] = 0.f;
#pragma unroll
    for (int i = 0; i < NP; ++i) pacc[i] = 0.f;
    int nxt = (gl < end - beg) ? __ldcs(a.nbr + beg + gl) : 0;   // index prefetch (gcn.cu)
    for (int base = beg; base < end; base += RL) {
        const int n = min(RL, end - base);
        const int my = nxt;
        nxt = (gl < end - base - RL) ? __ldcs(a.nbr + base + RL + gl) : 0;
#pragma unroll
        for (int j0 = 0; j0 < L; j0 += UB) {
            if (j0 * S >= n) break;
            float z[UB], x[UB][NV];
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) {
                const int k = (j0 + jj) * S + slot;
                const int u = __shfl_sync(gmask, my, k & (RL - 1), RL);
                if (k < n && j0 + jj < L) {
                    z[jj] = lrelu(__ldg(a.el + u) + erv, a.slope);
                    load_chunks<VPL>(a.T + (int64_t)u * a.ld, col0, W, x[jj]);
                } else {
                    z[jj] = -INFINITY;
#pragma unroll
                    for (int i = 0; i < NV; ++i) x[jj][i] = 0.f;
                }
            }
            float mb = m;
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) mb = fmaxf(mb, z[jj]);
            if (mb > m) {
                const float corr = (m == -INFINITY) ? 0.f : expf(m - mb);
                ssum *= corr;
#pragma unroll
                for (int i = 0; i < NV; ++i) acc[i] *= corr;
                if (SB) {
                    psum *= corr;
#pragma unroll
                    for (int i = 0; i < NP; ++i) pacc[i] *= corr;
                }
                m = mb;
            }
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) {
                const float p = (z[jj] == -INFINITY) ? 0.f : expf(z[jj] - m);
                ssum += p;
#pragma unroll
                for (int i = 0; i < NV; ++i) acc[i] = fmaf(p, x[jj][i], acc[i]);
                if (SB) {
                    const float pp = z[jj] > 0.f ? p : 0.f;
                    psum += pp;
#pragma unroll
                    for (int i = 0; i < NP; ++i) pacc[i] = fmaf(pp, x[jj][i % NV], pacc[i]);
                }
            }
        }
    }
#pragma unroll
    for (int o = L; o < RL; o <<= 1) {
        const float mo = __shfl_xor_sync(gmask, m, o, RL);
        const float so = __shfl_xor_sync(gmask, ssum, o, RL);
        const float mn = fmaxf(m, mo);
        const float ca = (m == -INFINITY) ? 0.f : expf(m - mn);
        const float cb = (mo == -INFINITY) ? 0.f : expf(mo - mn);
        ssum = ssum * ca + so * cb;
#pragma unroll
        for (int i = 0; i < NV; ++i) acc[i] = acc[i] * ca + __shfl_xor_sync(gmask, acc[i], o, RL) * cb;
        if (SB) {
            psum = psum * ca + __shfl_xor_sync(gmask, psum, o, RL) * cb;
#pragma unroll
            for (int i = 0; i < NP; ++i) pacc[i] = pacc[i] * ca + __shfl_xor_sync(gmask, pacc[i], o, RL) * cb;
        }
        m = mn;
    }
    if (!valid || slot != 0) return;
    const float inv = ssum > 0.f ? 1.f / ssum : 0.f;
    float* pa = a.A + v * a.ld;
    float* py = a.Y + v * a.ld;
    float* pb = SB ? a.B + v * a.ld : nullptr;
#pragma unroll
    for (int q = 0; q < VPL; ++q) {
        const int col = col0 + 4 * q;
        if (col >= W) continue;
        float o4[4], y4[4], b4[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            o4[i] = acc[4 * q + i] * inv;
            y4[i] = act_apply(a.act, o4[i] + ((a.bias && col + i < W) ? __ldg(a.bias + col + i) : 0.f));
            b4[i] = SB ? a.slope * o4[i] + (1.f - a.slope) * pacc[(4 * q + i) % NP] * inv : 0.f;
        }
        if (col + 4 <= W) {
            *reinterpret_cast<float4*>(pa + col) = make_float4(o4[0], o4[1], o4[2], o4[3]);
            *reinterpret_cast<float4*>(py + col) = make_float4(y4[0], y4[1], y4[2], y4[3]);
            if (SB) *reinterpret_cast<float4*>(pb + col) = make_float4(b4[0], b4[1], b4[2], b4[3]);
        } else {
            for (int i = 0; i < 4 && col + i < W; ++i) {
                pa[col + i] = o4[i];
                py[col + i] = y4[i];
                if (SB) pb[col + i] = b4[i];
            }
        }
    }
    if (c == 0) {
        a.lse[v] = ssum > 0.f ? m + logf(ssum) : -INFINITY;
        if (SB) a.bsum[v] = ssum > 0.f ? a.slope + (1.f - a.slope) * psum * inv : 0.f;
    }
}

// DER = false: source-major dT/del over REV; DER = true: destination-major der over FWD
template <int VPL, int L, int RL, bool DER>
__global__ void __launch_bounds__(256, GAT_MB_BWD) k_gat_bwd_h1(const GatBwdArgs a) {
    constexpr int NV = 4 * VPL, S = RL / L, UB = VPL <= 2 ? 4 : 2;
    const int lane = threadIdx.x & 31;
    const int gl = lane % RL, slot = gl / L, c = gl % L;
    const unsigned gmask = (RL == 32) ? 0xffffffffu : (((1u << RL) - 1u) << ((lane / RL) * RL));
    const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t row = a.row_begin + warp * (32 / RL) + lane / RL;
    const bool valid = row < a.row_end;
    const int beg = valid ? __ldg(a.off + row) : 0;
    const int end = valid ? __ldg(a.off + row + 1) : 0;
    const int64_t w = valid ? (int64_t)__ldg(a.perm + row) - a.vbase : 0;   // u (src-major) or v (der)
    const int W = a.F, col0 = c * NV;
    const int aux0 = rec_aux_offset(W);
    // per-row constants: src-major holds T_u and el_u; der holds dA_v and (er, lse, c)_v
    float own[NV];
    float k0 = 0.f, k1 = 0.f, k2 = 0.f;
    if (valid) {
        if (!DER) {
            load_chunks<VPL>(a.T + w * a.ldt, col0, W, own);
            k0 = __ldg(a.el + w);
        } else {
            const float* rec = a.D + w * a.ldd;
            load_chunks<VPL>(rec, col0, W, own);
            k0 = __ldg(rec + aux0); k1 = __ldg(rec + aux0 + 1); k2 = __ldg(rec + aux0 + 2);
        }
    } else {
#pragma unroll
        for (int i = 0; i < NV; ++i) own[i] = 0.f;
    }
    float acc[NV], dsum = 0.f;
#pragma unroll
    for (int i = 0; i < NV; ++i) acc[i] = 0.f;
    int nxt = (gl < end - beg) ? __ldcs(a.nbr + beg + gl) : 0;   // index prefetch (gcn.cu)
    for (int base = beg; base < end; base += RL) {
        const int n = min(RL, end - base);
        const int my = nxt;
        nxt = (gl < end - base - RL) ? __ldcs(a.nbr + base + RL + gl) : 0;
#pragma unroll
        for (int j0 = 0; j0 < L; j0 += UB) {
            if (j0 * S >= n) break;
            float x[UB][NV], e0[UB], e1[UB], e2[UB];
            bool ok[UB];
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) {
                const int k = (j0 + jj) * S + slot;
                const int o = __shfl_sync(gmask, my, k & (RL - 1), RL);
                ok[jj] = k < n && j0 + jj < L;
                if (ok[jj]) {
                    if (!DER) {
                        const float* rec = a.D + (int64_t)o * a.ldd;
                        load_chunks<VPL>(rec, col0, W, x[jj]);
                        const float4 ax = ldg4(rec + aux0);
                        e0[jj] = ax.x; e1[jj] = ax.y; e2[jj] = ax.z;
                    } else {
                        load_chunks<VPL>(a.T + (int64_t)o * a.ldt, col0, W, x[jj]);
                        e0[jj] = __ldg(a.el + o);
                        e1[jj] = 0.f; e2[jj] = 0.f;
                    }
                } else {
#pragma unroll
                    for (int i = 0; i < NV; ++i) x[jj][i] = 0.f;
                    e0[jj] = 0.f; e1[jj] = INFINITY; e2[jj] = 0.f;
                }
            }
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) {
                float g = 0.f;
#pragma unroll
                for (int i = 0; i < NV; ++i) g = fmaf(x[jj][i], own[i], g);
#pragma unroll
                for (int o = 1; o < L; o <<= 1) g += __shfl_xor_sync(gmask, g, o, RL);
                if (!ok[jj]) continue;
                // s = el_u + er_v ; alpha = exp(LReLU(s) - lse_v) ; ds = alpha (g - c_v) LReLU'(s)
                const float s = DER ? e0[jj] + k0 : k0 + e0[jj];
                const float lse = DER ? k1 : e1[jj];
                const float cv = DER ? k2 : e2[jj];
                const float al = expf(lrelu(s, a.slope) - lse);
                dsum += al * (g - cv) * (s > 0.f ? 1.f : a.slope);
                if (!DER) {
#pragma unroll
                    for (int i = 0; i < NV; ++i) acc[i] = fmaf(al, x[jj][i], acc[i]);
                }
            }
        }
    }
#pragma unroll
    for (int o = L; o < RL; o <<= 1) {
        if (!DER) {
#pragma unroll
            for (int i = 0; i < NV; ++i) acc[i] += __shfl_xor_sync(gmask, acc[i], o, RL);
        }
        dsum += __shfl_xor_sync(gmask, dsum, o, RL);
    }
    if (!valid || slot != 0) return;
    if (DER) {
        if (c == 0) a.der[w] = dsum;
        return;
    }
    float* pd = a.dT + w * a.ldt;
#pragma unroll
    for (int q = 0; q < VPL; ++q) {
        const int col = col0 + 4 * q;
        if (col >= W) continue;
        if (col + 4 <= W)
            *reinterpret_cast<float4*>(pd + col) = make_float4(acc[4 * q], acc[4 * q + 1], acc[4 * q + 2], acc[4 * q + 3]);
        else
            for (int i = 0; i < 4 && col + i < W; ++i) pd[col + i] = acc[4 * q + i];
    }
    if (c == 0) a.del[w] = dsum;
}

// ============================================================================================
// row kernels
// ============================================================================================
// thread per (u,h): el/er projections
__global__ void k_gat_attn_proj(const float* __restrict__ T, int64_t M, int H, int F, int64_t ldt,
                                const float* __restrict__ a_l, const float* __restrict__ a_r, float* __restrict__ el,
                                float* __restrict__ er) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i >= M * H) return;
    const int64_t u = i / H;
    const int h = (int)(i % H);
    const float* t = T + u * ldt + (int64_t)h * F;
    float sl = 0.f, sr = 0.f;
    for (int f = 0; f < F; ++f) {
        const float x = __ldg(t + f);
        sl = fmaf(x, __ldg(a_l + h * F + f), sl);
        sr = fmaf(x, __ldg(a_r + h * F + f), sr);
    }
    if (el) el[i] = sl;
    if (er) er[i] = sr;
}

// thread per (v,h): dA = dY act'(Y), c = <dA, A>, record D[v] = [dA | (er, lse, c, 0) per head]
__global__ void k_gat_bwd_prep(int64_t M, int H, int F, int64_t ldt, const float* __restrict__ dY,
                               const float* __restrict__ Y, int act, const float* __restrict__ A,
                               const float* __restrict__ er, const float* __restrict__ lse, float* __restrict__ D,
                               int64_t ldd, const float* __restrict__ B, const float* __restrict__ bsum,
                               float* __restrict__ der) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i >= M * H) return;
    const int64_t v = i / H;
    const int h = (int)(i % H);
    const int64_t o = v * ldt + (int64_t)h * F;
    float* rec = D + v * ldd;
    float cdot = 0.f, bdot = 0.f;
    for (int f = 0; f < F; ++f) {
        float d = __ldg(dY + o + f);
        if (act != SEASTAR_ACT_NONE) d *= act_grad_from_y(act, __ldg(Y + o + f));
        rec[(int64_t)h * F + f] = d;
        cdot = fmaf(d, __ldg(A + o + f), cdot);
        if (B) bdot = fmaf(d, __ldg(B + o + f), bdot);
    }
    // der_v = sum_e a_e LReLU'(s_e) (g_e - c_v) = <dA_v, B_v> - c_v b_v   (B, b from the forward)
    if (B) der[i] = bdot - cdot * __ldg(bsum + i);
    if (h == H - 1)   // zero the padding between dA and the aux block so vector loads read zeros
        for (int64_t f = (int64_t)H * F; f < rec_aux_offset(H * F); ++f) rec[f] = 0.f;
    float* aux = rec + rec_aux_offset(H * F) + 4 * h;
    aux[0] = __ldg(er + i);
    aux[1] = __ldg(lse + i);
    aux[2] = cdot;
    aux[3] = 0.f;
}

// stage 1 of attn_proj_bwd: dT += del a_l + der a_r (in place) and per-block partial da_l, da_r
__global__ void __launch_bounds__(256) k_gat_attn_proj_bwd1(const float* __restrict__ T, int64_t M, int H, int F,
                                                            int64_t ldt, const float* __restrict__ a_l,
                                                            const float* __restrict__ a_r,
                                                            const float* __restrict__ del,
                                                            const float* __restrict__ der, float* __restrict__ dT,
                                                            int64_t rows_per_block, float* __restrict__ part) {
    const int W = H * F;
    const int64_t r0 = blockIdx.x * rows_per_block;
    const int64_t r1 = min(M, r0 + rows_per_block);
    __shared__ float red[2][8][33];
    float* pl = part + (int64_t)blockIdx.x * 2 * W;
    for (int cb = 0; cb < W; cb += 32) {
        const int j = cb + (threadIdx.x & 31);
        const int ty = threadIdx.x >> 5;          // 8 row lanes
        float sl = 0.f, sr = 0.f;
        if (j < W) {
            const int h = j / F;
            const float al = __ldg(a_l + j), ar = __ldg(a_r + j);
            for (int64_t r = r0 + ty; r < r1; r += 8) {
                const float t = __ldg(T + r * ldt + j);
                const float dl = del ? __ldg(del + r * H + h) : 0.f;
                const float dr = der ? __ldg(der + r * H + h) : 0.f;
                dT[r * ldt + j] += dl * al + dr * ar;
                sl = fmaf(dl, t, sl);
                sr = fmaf(dr, t, sr);
            }
        }
        red[0][ty][threadIdx.x & 31] = sl;
        red[1][ty][threadIdx.x & 31] = sr;
        __syncthreads();
        if (ty < 2 && j < W) {
            float x = 0.f;
            for (int k = 0; k < 8; ++k) x += red[ty][k][threadIdx.x & 31];
            pl[ty * W + j] = x;
        }
        __syncthreads();
    }
}

// stage 2: out[j] = sum_b part[b*stride + j] in block order
__global__ void k_sum_partials(const float* __restrict__ part, int64_t nblk, int64_t stride, int64_t n,
                               float* __restrict__ out) {
    const int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (j >= n) return;
    float x = 0.f;
    for (int64_t b = 0; b < nblk; ++b) x += part[b * stride + j];
    out[j] = x;
}

static int64_t proj_bwd_blocks(int64_t M) {
    int64_t b = 2 * num_sms();
    if (M < b * 64) b = (M + 63) / 64;
    return b < 1 ? 1 : b;
}

// ============================================================================================
// launch helpers
// ============================================================================================
// head-per-lane applies when every head row is whole float4s held by one lane
static int hpl_f4(int H, int F, int64_t ldt, bool aligned) {
    if (H < 2 || (32 % H) != 0 || (F % 4) != 0 || F > 32 || (ldt % 4) != 0 || !aligned) return 0;
    return F / 4;
}


#define SS_HPL_SWITCH(KERNEL, f4, grid, s, args)                      \
    switch (f4) {                                                     \
        case 1: launch_k(KERNEL<1>, dim3(grid), dim3(256), 0, s, args); break;          \
        case 2: launch_k(KERNEL<2>, dim3(grid), dim3(256), 0, s, args); break;          \
        case 3: launch_k(KERNEL<3>, dim3(grid), dim3(256), 0, s, args); break;          \
        case 4: launch_k(KERNEL<4>, dim3(grid), dim3(256), 0, s, args); break;          \
        case 5: launch_k(KERNEL<5>, dim3(grid), dim3(256), 0, s, args); break;          \
        case 6: launch_k(KERNEL<6>, dim3(grid), dim3(256), 0, s, args); break;          \
        case 7: launch_k(KERNEL<7>, dim3(grid), dim3(256), 0, s, args); break;          \
        default: launch_k(KERNEL<8>, dim3(grid), dim3(256), 0, s, args); break;         \
    }

#define SS_HPL_SWITCH_SB(KERNEL, SB, f4, grid, s, args)                          \
    switch (f4) {                                                                 \
        case 1: launch_k(KERNEL<1, SB>, dim3(grid), dim3(256), 0, s, args); break; \
        case 2: launch_k(KERNEL<2, SB>, dim3(grid), dim3(256), 0, s, args); break; \
        case 3: launch_k(KERNEL<3, SB>, dim3(grid), dim3(256), 0, s, args); break; \
        case 4: launch_k(KERNEL<4, SB>, dim3(grid), dim3(256), 0, s, args); break; \
        case 5: launch_k(KERNEL<5, SB>, dim3(grid), dim3(256), 0, s, args); break; \
        case 6: launch_k(KERNEL<6, SB>, dim3(grid), dim3(256), 0, s, args); break; \
        case 7: launch_k(KERNEL<7, SB>, dim3(grid), dim3(256), 0, s, args); break; \
        default: launch_k(KERNEL<8, SB>, dim3(grid), dim3(256), 0, s, args); break; \
    }

#define SS_CHUNK_SWITCH(KERNEL, VEC, L, RL, grid, s, args)            \
    switch (L) {                                                      \
        case 1: launch_k(KERNEL<VEC, 1, 32>, dim3(grid), dim3(256), 0, s, args); break; \
        case 2: launch_k(KERNEL<VEC, 2, 32>, dim3(grid), dim3(256), 0, s, args); break; \
        case 4: launch_k(KERNEL<VEC, 4, RL>, dim3(grid), dim3(256), 0, s, args); break; \
        case 8: launch_k(KERNEL<VEC, 8, RL>, dim3(grid), dim3(256), 0, s, args); break; \
        case 16: launch_k(KERNEL<VEC, 16, RL>, dim3(grid), dim3(256), 0, s, args); break; \
        default: launch_k(KERNEL<VEC, 32, 32>, dim3(grid), dim3(256), 0, s, args); break; \
    }

// chunked launches over the two degree classes: warp rows (RL = 32) and sub-warp rows (RL = L)
template <typename Args, typename LaunchWarp, typename LaunchSub>
static void two_buckets(Args a, int64_t split, int64_t n_rows, int L, LaunchWarp lw, LaunchSub ls) {
    Args hi = a, lo = a;
    hi.row_begin = 0; hi.row_end = split;
    lo.row_begin = split; lo.row_end = n_rows;
    if (split > 0) lw(hi, (unsigned)((split + 7) / 8));
    if (n_rows > split) {
        const int RL = L < 4 ? 4 : L;
        const int64_t per = 256 / RL;
        ls(lo, (unsigned)((n_rows - split + per - 1) / per));
    }
}

// single-head path: VPL chunks per lane (from {1,2,3,4,6,8}) and L = pow2 lanes per edge (<= 4)
static bool h1_geometry(int H, int F, int64_t ldt, bool aligned, int& vpl, int& L) {
    if (H != 1 || (ldt % 4) != 0 || !aligned || F > 128) return false;
    const int C = (F + 3) / 4;
    int v = (C + 3) / 4;
    v = v <= 4 ? v : (v <= 6 ? 6 : 8);
    vpl = v;
    L = pow2_ceil((C + v - 1) / v);
    return L <= 4;
}

struct FwdH1 {
    template <int VPL, int L>
    static void run(const GatFwdArgs& a, int64_t split, int64_t n, cudaStream_t s) {
        if (a.B)
            two_buckets(a, split, n, 4,
                        [&](GatFwdArgs x, unsigned grid) { launch_k(k_gat_fwd_h1<VPL, L, 32, true>, dim3(grid), dim3(256), 0, s, x); },
                        [&](GatFwdArgs x, unsigned grid) { launch_k(k_gat_fwd_h1<VPL, L, 4, true>, dim3(grid), dim3(256), 0, s, x); });
        else
            two_buckets(a, split, n, 4,
                        [&](GatFwdArgs x, unsigned grid) { launch_k(k_gat_fwd_h1<VPL, L, 32, false>, dim3(grid), dim3(256), 0, s, x); },
                        [&](GatFwdArgs x, unsigned grid) { launch_k(k_gat_fwd_h1<VPL, L, 4, false>, dim3(grid), dim3(256), 0, s, x); });
    }
};
template <bool DER>
struct BwdH1 {
    template <int VPL, int L>
    static void run(const GatBwdArgs& a, int64_t split, int64_t n, cudaStream_t s) {
        two_buckets(a, split, n, 4,
                    [&](GatBwdArgs x, unsigned grid) { launch_k(k_gat_bwd_h1<VPL, L, 32, DER>, dim3(grid), dim3(256), 0, s, x); },
                    [&](GatBwdArgs x, unsigned grid) { launch_k(k_gat_bwd_h1<VPL, L, 4, DER>, dim3(grid), dim3(256), 0, s, x); });
    }
};
template <class K, int VPL, class Args>
static void dispatch_h1_L(int L, const Args& a, int64_t split, int64_t n, cudaStream_t s) {
    switch (L) {
        case 1: K::template run<VPL, 1>(a, split, n, s); break;
        case 2: K::template run<VPL, 2>(a, split, n, s); break;
        default: K::template run<VPL, 4>(a, split, n, s); break;
    }
}
template <class K, class Args>
static void dispatch_h1(int vpl, int L, const Args& a, int64_t split, int64_t n, cudaStream_t s) {
    switch (vpl) {
        case 1: dispatch_h1_L<K, 1>(L, a, split, n, s); break;
        case 2: dispatch_h1_L<K, 2>(L, a, split, n, s); break;
        case 3: dispatch_h1_L<K, 3>(L, a, split, n, s); break;
        case 4: dispatch_h1_L<K, 4>(L, a, split, n, s); break;
        case 6: dispatch_h1_L<K, 6>(L, a, split, n, s); break;
        default: dispatch_h1_L<K, 8>(L, a, split, n, s); break;
    }
}

}  // namespace seastar

using namespace seastar;

#define CHUNK_LAUNCH(KERNEL, ARGS, SPLIT, NROWS, L, VEC4, S)                                                     \
    do {                                                                                                         \
        auto lw = [&](decltype(ARGS) x, unsigned grid) {                                                         \
            if (VEC4) { SS_CHUNK_SWITCH(KERNEL, 4, L, 32, grid, S, x); }                                         \
            else { SS_CHUNK_SWITCH(KERNEL, 1, L, 32, grid, S, x); }                                              \
        };                                                                                                       \
        auto ls = [&](decltype(ARGS) x, unsigned grid) {                                                         \
            if (VEC4) {                                                                                          \
                switch (L) {                                                                                     \
                    case 1: launch_k(KERNEL<4, 1, 4>, dim3(grid), dim3(256), 0, S, x); break;                                      \
                    case 2: launch_k(KERNEL<4, 2, 4>, dim3(grid), dim3(256), 0, S, x); break;                                      \
                    case 4: launch_k(KERNEL<4, 4, 4>, dim3(grid), dim3(256), 0, S, x); break;                                      \
                    case 8: launch_k(KERNEL<4, 8, 8>, dim3(grid), dim3(256), 0, S, x); break;                                      \
                    case 16: launch_k(KERNEL<4, 16, 16>, dim3(grid), dim3(256), 0, S, x); break;                                   \
                    default: launch_k(KERNEL<4, 32, 32>, dim3(grid), dim3(256), 0, S, x); break;                                   \
                }                                                                                                \
            } else {                                                                                             \
                switch (L) {                                                                                     \
                    case 1: launch_k(KERNEL<1, 1, 4>, dim3(grid), dim3(256), 0, S, x); break;                                      \
                    case 2: launch_k(KERNEL<1, 2, 4>, dim3(grid), dim3(256), 0, S, x); break;                                      \
                    case 4: launch_k(KERNEL<1, 4, 4>, dim3(grid), dim3(256), 0, S, x); break;                                      \
                    case 8: launch_k(KERNEL<1, 8, 8>, dim3(grid), dim3(256), 0, S, x); break;                                      \
                    case 16: launch_k(KERNEL<1, 16, 16>, dim3(grid), dim3(256), 0, S, x); break;                                   \
                    default: launch_k(KERNEL<1, 32, 32>, dim3(grid), dim3(256), 0, S, x); break;                                   \
                }                                                                                                \
            }                                                                                                    \
        };                                                                                                       \
        two_buckets(ARGS, (L) >= 32 ? (NROWS) : (SPLIT), NROWS, L, lw, ls);                                      \
    } while (0)

extern "C" {

int64_t seastar_gat_record_ld(int32_t H, int32_t F) { return ((int64_t)H * F + 3) / 4 * 4 + 4 * (int64_t)H; }

seastar_status seastar_gat_attn_proj(const float* T, int64_t M, int32_t H, int32_t F, int64_t ldt, const float* a_l,
                                     const float* a_r, float* el, float* er, seastar_stream stream) {
    SS_ARG(T && a_l && a_r && (el || er), "gat_attn_proj: NULL argument");
    SS_ARG(M >= 0 && H >= 1 && F >= 1 && ldt >= (int64_t)H * F, "gat_attn_proj: bad sizes");
    SS_TRY(check_device());
    if (M == 0) return SEASTAR_OK;
    const int64_t n = M * H;
    k_gat_attn_proj<<<(unsigned)((n + 255) / 256), 256, 0, to_stream(stream)>>>(T, M, H, F, ldt, a_l, a_r, el, er);
    return check_launch("k_gat_attn_proj");
}

seastar_status seastar_gat_fwd(seastar_graph g, const float* T_all, const float* el_all, const float* er_loc,
                               int32_t H, int32_t F, int64_t ldt, float slope, const float* bias, seastar_act act,
                               float* A_loc, float* Y_loc, float* lse_loc, float* B_loc, float* b_loc,
                               seastar_stream stream) {
    SS_ARG(g && T_all && el_all && er_loc && A_loc && Y_loc && lse_loc, "gat_fwd: NULL argument");
    SS_ARG((B_loc == nullptr) == (b_loc == nullptr), "gat_fwd: pass both B_loc and b_loc or neither");
    SS_ARG(!B_loc || (aligned16(B_loc) == aligned16(A_loc)), "gat_fwd: B_loc must be aligned like A_loc");
    SS_ARG(H >= 1 && F >= 1 && ldt >= (int64_t)H * F, "gat_fwd: bad sizes H=%d F=%d ldt=%lld", H, F, (long long)ldt);
    SS_ARG(act >= SEASTAR_ACT_NONE && act <= SEASTAR_ACT_SIGMOID, "gat_fwd: bad activation");
    SS_TRY(check_device());
    cudaStream_t s = to_stream(stream);
    GatFwdArgs a{};
    a.perm = g->fwd.perm; a.off = g->fwd.off; a.nbr = g->fwd.nbr;
    a.vbase = g->row_begin;
    a.T = T_all; a.el = el_all; a.er = er_loc;
    a.H = H; a.F = F; a.ld = ldt; a.slope = slope; a.bias = bias; a.act = act;
    a.A = A_loc; a.Y = Y_loc; a.lse = lse_loc; a.B = B_loc; a.bsum = b_loc;
    const int f4 = hpl_f4(H, F, ldt, aligned16(T_all) && aligned16(A_loc) && aligned16(Y_loc));
    if (f4) {
        a.row_begin = 0; a.row_end = g->fwd.n_rows;
        const unsigned grid = (unsigned)((g->fwd.n_rows + 7) / 8);
        if (grid && a.B) SS_HPL_SWITCH_SB(k_gat_fwd_hpl, true, f4, grid, s, a);
        if (grid && !a.B) SS_HPL_SWITCH_SB(k_gat_fwd_hpl, false, f4, grid, s, a);
        return check_launch("k_gat_fwd_hpl");
    }
    int vpl = 0, Lh = 0;
    if (h1_geometry(H, F, ldt, aligned16(T_all) && aligned16(A_loc) && aligned16(Y_loc), vpl, Lh)) {
        dispatch_h1<FwdH1>(vpl, Lh, a, g->fwd.bucket_rows[1], g->fwd.n_rows, s);
        return check_launch("k_gat_fwd_h1");
    }
    const bool vec4 = (ldt % 4 == 0) && (H == 1 || F % 4 == 0) && aligned16(T_all) && aligned16(A_loc) &&
                      aligned16(Y_loc);
    const int VEC = vec4 ? 4 : 1;
    const int C = (H * F + VEC - 1) / VEC;
    SS_ARG(C <= 32, "gat_fwd: row of H*F=%d floats exceeds 32 lanes x %d", H * F, VEC);
    const int L = pow2_ceil(C);
    CHUNK_LAUNCH(k_gat_fwd, a, g->fwd.bucket_rows[1], g->fwd.n_rows, L, vec4, s);
    return check_launch("k_gat_fwd");
}

seastar_status seastar_gat_bwd_prep(seastar_graph g, const float* dY_loc, const float* Y_loc, seastar_act act,
                                    const float* A_loc, const float* er_loc, const float* lse_loc, int32_t H,
                                    int32_t F, int64_t ldt, float* D_loc, const float* B_loc, const float* b_loc,
                                    float* der_loc, seastar_stream stream) {
    SS_ARG(g && dY_loc && A_loc && er_loc && lse_loc && D_loc, "gat_bwd_prep: NULL argument");
    SS_ARG((B_loc == nullptr) == (b_loc == nullptr) && (B_loc == nullptr) == (der_loc == nullptr),
           "gat_bwd_prep: pass B_loc, b_loc and der_loc together or none of them");
    SS_ARG(act == SEASTAR_ACT_NONE || Y_loc, "gat_bwd_prep: Y_loc is required for act != NONE");
    SS_ARG(H >= 1 && F >= 1 && ldt >= (int64_t)H * F, "gat_bwd_prep: bad sizes");
    SS_TRY(check_device());
    const int64_t M = g->n_loc();
    if (M == 0) return SEASTAR_OK;
    const int64_t n = M * H;
    k_gat_bwd_prep<<<(unsigned)((n + 255) / 256), 256, 0, to_stream(stream)>>>(
        M, H, F, ldt, dY_loc, Y_loc, act, A_loc, er_loc, lse_loc, D_loc, seastar_gat_record_ld(H, F), B_loc, b_loc,
        der_loc);
    return check_launch("k_gat_bwd_prep");
}

seastar_status seastar_gat_bwd(seastar_graph g, const float* T_loc, const float* el_loc, const float* D_all,
                               int32_t H, int32_t F, int64_t ldt, float slope, float* dT_loc, float* del_loc,
                               seastar_stream stream) {
    SS_ARG(g && T_loc && el_loc && D_all && dT_loc && del_loc, "gat_bwd: NULL argument");
    SS_ARG(H >= 1 && F >= 1 && ldt >= (int64_t)H * F, "gat_bwd: bad sizes");
    SS_TRY(check_device());
    cudaStream_t s = to_stream(stream);
    GatBwdArgs a{};
    a.perm = g->rev.perm; a.off = g->rev.off; a.nbr = g->rev.nbr;
    a.vbase = g->row_begin;
    a.T = T_loc; a.el = el_loc; a.D = D_all;
    a.H = H; a.F = F; a.ldt = ldt; a.ldd = seastar_gat_record_ld(H, F); a.slope = slope;
    a.dT = dT_loc; a.del = del_loc;
    ScopedL2Window win(D_all, (size_t)g->N * a.ldd * sizeof(float));
    const int f4 = hpl_f4(H, F, ldt, aligned16(T_loc) && aligned16(D_all) && aligned16(dT_loc));
    if (f4) {
        a.row_begin = 0; a.row_end = g->rev.n_rows;
        const unsigned grid = (unsigned)((g->rev.n_rows + 7) / 8);
        if (grid) SS_HPL_SWITCH(k_gat_bwd_hpl, f4, grid, s, a);
        return check_launch("k_gat_bwd_hpl");
    }
    int vpl = 0, Lh = 0;
    if (h1_geometry(H, F, ldt, aligned16(T_loc) && aligned16(D_all) && aligned16(dT_loc), vpl, Lh)) {
        dispatch_h1<BwdH1<false>>(vpl, Lh, a, g->rev.bucket_rows[1], g->rev.n_rows, s);
        return check_launch("k_gat_bwd_h1");
    }
    const bool vec4 = (ldt % 4 == 0) && (H == 1 || F % 4 == 0) && aligned16(T_loc) && aligned16(D_all) &&
                      aligned16(dT_loc);
    const int VEC = vec4 ? 4 : 1;
    const int C = (H * F + VEC - 1) / VEC;
    SS_ARG(C <= 32, "gat_bwd: row of H*F=%d floats exceeds 32 lanes x %d", H * F, VEC);
    const int L = pow2_ceil(C);
    CHUNK_LAUNCH(k_gat_bwd, a, g->rev.bucket_rows[1], g->rev.n_rows, L, vec4, s);
    return check_launch("k_gat_bwd");
}

seastar_status seastar_gat_der(seastar_graph g, const float* T_all, const float* el_all, const float* D_loc, int32_t H,
                               int32_t F, int64_t ldt, float slope, float* der_loc, seastar_stream stream) {
    SS_ARG(g && T_all && el_all && D_loc && der_loc, "gat_der: NULL argument");
    SS_ARG(H >= 1 && F >= 1 && ldt >= (int64_t)H * F, "gat_der: bad sizes");
    SS_TRY(check_device());
    cudaStream_t s = to_stream(stream);
    GatBwdArgs a{};
    a.perm = g->fwd.perm; a.off = g->fwd.off; a.nbr = g->fwd.nbr;
    a.vbase = g->row_begin;
    a.T = T_all; a.el = el_all; a.D = D_loc;
    a.H = H; a.F = F; a.ldt = ldt; a.ldd = seastar_gat_record_ld(H, F); a.slope = slope;
    a.der = der_loc;
    const int f4 = hpl_f4(H, F, ldt, aligned16(T_all) && aligned16(D_loc));
    if (f4) {
        a.row_begin = 0; a.row_end = g->fwd.n_rows;
        const unsigned grid = (unsigned)((g->fwd.n_rows + 7) / 8);
        if (grid) SS_HPL_SWITCH(k_gat_der_hpl, f4, grid, s, a);
        return check_launch("k_gat_der_hpl");
    }
    int vpl = 0, Lh = 0;
    if (h1_geometry(H, F, ldt, aligned16(T_all) && aligned16(D_loc), vpl, Lh)) {
        dispatch_h1<BwdH1<true>>(vpl, Lh, a, g->fwd.bucket_rows[1], g->fwd.n_rows, s);
        return check_launch("k_gat_der_h1");
    }
    const bool vec4 = (ldt % 4 == 0) && (H == 1 || F % 4 == 0) && aligned16(T_all) && aligned16(D_loc);
    const int VEC = vec4 ? 4 : 1;
    const int C = (H * F + VEC - 1) / VEC;
    SS_ARG(C <= 32, "gat_der: row of H*F=%d floats exceeds 32 lanes x %d", H * F, VEC);
    const int L = pow2_ceil(C);
    CHUNK_LAUNCH(k_gat_der, a, g->fwd.bucket_rows[1], g->fwd.n_rows, L, vec4, s);
    return check_launch("k_gat_der");
}

size_t seastar_gat_attn_proj_bwd_workspace(int64_t M, int32_t H, int32_t F) {
    return (size_t)proj_bwd_blocks(M) * 2 * (size_t)H * F * sizeof(float) + 256;
}

seastar_status seastar_gat_attn_proj_bwd(const float* T, int64_t M, int32_t H, int32_t F, int64_t ldt,
                                         const float* a_l, const float* a_r, const float* del, const float* der,
                                         float* dT, float* da_l, float* da_r, void* workspace, size_t ws_bytes,
                                         seastar_stream stream) {
    SS_ARG(T && a_l && a_r && dT && da_l && da_r && workspace, "gat_attn_proj_bwd: NULL argument");
    SS_ARG(M >= 0 && H >= 1 && F >= 1 && ldt >= (int64_t)H * F, "gat_attn_proj_bwd: bad sizes");
    SS_ARG(ws_bytes >= seastar_gat_attn_proj_bwd_workspace(M, H, F), "gat_attn_proj_bwd: workspace too small");
    SS_TRY(check_device());
    cudaStream_t s = to_stream(stream);
    const int W = H * F;
    const int64_t nblk = proj_bwd_blocks(M);
    const int64_t rpb = (M + nblk - 1) / nblk;
    float* part = static_cast<float*>(workspace);
    k_gat_attn_proj_bwd1<<<(unsigned)nblk, 256, 0, s>>>(T, M, H, F, ldt, a_l, a_r, del, der, dT, rpb > 0 ? rpb : 1, part);
    k_sum_partials<<<(unsigned)((W + 255) / 256), 256, 0, s>>>(part, nblk, 2 * (int64_t)W, W, da_l);
    k_sum_partials<<<(unsigned)((W + 255) / 256), 256, 0, s>>>(part + W, nblk, 2 * (int64_t)W, W, da_r);
    return check_launch("k_gat_attn_proj_bwd");
}

}  // extern "C"
