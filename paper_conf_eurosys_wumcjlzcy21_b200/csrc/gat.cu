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
#include "gat_common.cuh"

namespace seastar {

#ifndef H1_MID_CLASS
#define H1_MID_CLASS 1   // single-head GAT rows with degree >= 2^(kPow2Lo + H1_MID_CLASS) = 8 take 16-lane row groups
#endif
constexpr int kH1MidClass = H1_MID_CLASS;

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
    const bool DROP = a.deid != nullptr;
    const uint64_t dkey = DROP ? drop_key(a.dseed, a.dsite, a.dstep) : 0ull;
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
            float z[UB], val[UB][VEC], mk[UB];
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) {
                const int k = (j0 + jj) * S + slot;
                const int u = __shfl_sync(gmask, my, k & (RL - 1), RL);
                mk[jj] = 1.f;
                if (k < n && active) {
                    z[jj] = lrelu(__ldg(a.el + (int64_t)u * a.ldel + h) + erv, a.slope);
                    load_vec<VEC>(a.T + (int64_t)u * a.ld + col, val[jj]);
                    if (DROP)
                        mk[jj] = drop_mult(dkey, (uint64_t)__ldg(a.deid + base + k) * a.H + h, a.dthr, a.dscale);
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
                const float pm = p * mk[jj], ppm = pp * mk[jj];     // attention dropout: weights only
#pragma unroll
                for (int i = 0; i < VEC; ++i) {
                    acc[i] = fmaf(pm, val[jj][i], acc[i]);
                    pacc[i] = fmaf(ppm, val[jj][i], pacc[i]);
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

// ============================================================================================
// backward
// ============================================================================================
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
    const float elu = (valid && active) ? __ldg(a.el + u * a.ldel + h) : 0.f;
    float acc[VEC], dl = 0.f;
#pragma unroll
    for (int i = 0; i < VEC; ++i) acc[i] = 0.f;
    const bool DROP = a.deid != nullptr;
    const uint64_t dkey = DROP ? drop_key(a.dseed, a.dsite, a.dstep) : 0ull;

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
                    const float mk =
                        DROP ? drop_mult(dkey, (uint64_t)__ldg(a.deid + base + k) * a.H + h, a.dthr, a.dscale) : 1.f;
                    dl += al * (mk * g - cv[jj]) * (s > 0.f ? 1.f : a.slope);
                    const float alm = al * mk;
#pragma unroll
                    for (int i = 0; i < VEC; ++i) acc[i] = fmaf(alm, dA[jj][i], acc[i]);
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
    const bool DROP = a.deid != nullptr;
    const uint64_t dkey = DROP ? drop_key(a.dseed, a.dsite, a.dstep) : 0ull;
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
                    elu[jj] = __ldg(a.el + (int64_t)u * a.ldel + h);
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
                    const float mk =
                        DROP ? drop_mult(dkey, (uint64_t)__ldg(a.deid + base + k) * a.H + h, a.dthr, a.dscale) : 1.f;
                    dr += al * (mk * g - cvv) * (s > 0.f ? 1.f : a.slope);
                }
            }
        }
    }
#pragma unroll
    for (int o = L; o < RL; o <<= 1) dr += __shfl_xor_sync(gmask, dr, o, RL);
    if (!valid || slot != 0 || !active) return;
    if (hc == 0) a.der[v * a.H + h] = dr;
}

// ============================================================================================
// row kernels
// ============================================================================================
// thread per (u,h): el/er projections
__global__ void k_gat_attn_proj(const float* __restrict__ T, int64_t M, int H, int F, int64_t ldt,
                                const float* __restrict__ a_l, const float* __restrict__ a_r, float* __restrict__ el,
                                float* __restrict__ er, int64_t ldel) {
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
    if (el) el[u * ldel + h] = sl;
    if (er) er[i] = sr;
}

// warp per row v (coalesced row reads): dA = dY act'(Y), c = <dA, A>, record D[v] = [dA | (er, lse, c, nl2)
// per head]; with the forward-saved factors also der_v = <dA_v, B_v> - c_v b_v.  c and der are carried in
// fp64: der cancels down to the LeakyReLU-negative part of the softmax (|der| << |c|).  Per-head sums are
// fixed xor trees (deterministic): segmented over the F lanes of a head when F divides 32, else one full
// warp reduction per head.
__device__ __forceinline__ double warp_sum_seg(double x, int width) {
    for (int o = width >> 1; o; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
    return x;
}

__global__ void __launch_bounds__(256) k_gat_bwd_prep(int64_t M, int H, int F, int64_t ldt,
                                                      const float* __restrict__ dY, const float* __restrict__ Y,
                                                      int act, const float* __restrict__ A,
                                                      const float* __restrict__ er, const float* __restrict__ lse,
                                                      float* __restrict__ D, int64_t ldd, const float* __restrict__ B,
                                                      const float* __restrict__ bsum, float* __restrict__ der) {
    const int lane = threadIdx.x & 31;
    const int64_t v = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    if (v >= M) return;
    const int W = H * F;
    const int64_t o = v * ldt;
    float* rec = D + v * ldd;
    const bool seg = (32 % F) == 0;           // a head's columns are F consecutive lanes of one 32-column pass
    double cdot = 0.0, bdot = 0.0;             // this lane's head (seg) -- valid after the reductions
    double cacc[8], bacc[8];                   // non-seg, H <= 8: per-head partials of this lane
#pragma unroll
    for (int h = 0; h < 8; ++h) cacc[h] = bacc[h] = 0.0;
    for (int j0 = 0; j0 < W; j0 += 32) {
        const int j = j0 + lane;
        double pc = 0.0, pb = 0.0;
        if (j < W) {
            float d = __ldg(dY + o + j);
            if (act != SEASTAR_ACT_NONE) d *= act_grad_from_y(act, __ldg(Y + o + j));
            rec[j] = d;
            pc = (double)d * (double)__ldg(A + o + j);
            if (B) pb = (double)d * (double)__ldg(B + o + j);
        }
        if (seg) {
            pc = warp_sum_seg(pc, F);
            pb = warp_sum_seg(pb, F);
            // every lane of head hh's group now holds its sum; lane hh (the head's owner, H <= 32) takes it
            for (int hh = j0 / F; hh < H && hh * F < j0 + 32; ++hh) {
                const double xc = __shfl_sync(0xffffffffu, pc, hh * F - j0);
                const double xb = __shfl_sync(0xffffffffu, pb, hh * F - j0);
                if (lane == hh) { cdot = xc; bdot = xb; }
            }
        } else {
            const int h = j < W ? j / F : 0;
#pragma unroll
            for (int hh = 0; hh < 8; ++hh)
                if (hh == h) { cacc[hh] += pc; bacc[hh] += pb; }
        }
    }
    if (!seg) {
#pragma unroll
        for (int hh = 0; hh < 8; ++hh) {
            if (hh >= H) break;
            const double xc = warp_sum_seg(cacc[hh], 32);
            const double xb = warp_sum_seg(bacc[hh], 32);
            if (lane == hh) { cdot = xc; bdot = xb; }
        }
    }
    // zero the padding between dA and the aux block so vector loads read zeros
    for (int f = W + lane; f < rec_aux_offset(W); f += 32) rec[f] = 0.f;
    if (lane < H) {
        const int64_t i = v * H + lane;
        if (B) der[i] = (float)(bdot - cdot * (double)__ldg(bsum + i));
        float* aux = rec + rec_aux_offset(W) + 4 * lane;
        aux[0] = __ldg(er + i);
        const float l = __ldg(lse + i);
        aux[1] = l;
        aux[2] = (float)cdot;
        aux[3] = -l * kLog2e;   // nl2: a_e = ex2(LReLU(s_e) log2 e + nl2)
    }
}

// vectorised row pass for the common geometry (W = H*F <= 128, float4-aligned rows, H == 1 or F/4 a power of
// two): LR = pow2(ceil(W/4)) lanes per row, one float4 chunk per lane, 32/LR rows per warp; per-head fp64 sums
// by a segmented xor tree over the lanes of the head (deterministic).  Same outputs as k_gat_bwd_prep.
template <int LR>
__global__ void __launch_bounds__(256) k_gat_bwd_prep4(int64_t M, int H, int F, int64_t ldt,
                                                       const float* __restrict__ dY, const float* __restrict__ Y,
                                                       int act, const float* __restrict__ A,
                                                       const float* __restrict__ er, const float* __restrict__ lse,
                                                       float* __restrict__ D, int64_t ldd, const float* __restrict__ B,
                                                       const float* __restrict__ bsum, float* __restrict__ der) {
    const int lane = threadIdx.x & 31;
    const int c = lane % LR;
    const int64_t v = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) / LR;
    const bool valid = v < M;
    const int W = H * F, C4 = (W + 3) / 4;
    const int lph = H == 1 ? LR : F / 4;                   // lanes per head (a power of two)
    const int h = H == 1 ? 0 : c / lph;
    double pc = 0.0, pb = 0.0;
    if (valid && c < C4) {
        const int64_t o = v * ldt + 4 * c;
        float d[4], y[4], a[4], b[4];
        const float4 dy = ldg4(dY + o);
        d[0] = dy.x; d[1] = dy.y; d[2] = dy.z; d[3] = dy.w;
        if (act != SEASTAR_ACT_NONE) {
            const float4 y4 = ldg4(Y + o);
            y[0] = y4.x; y[1] = y4.y; y[2] = y4.z; y[3] = y4.w;
#pragma unroll
            for (int i = 0; i < 4; ++i) d[i] *= act_grad_from_y(act, y[i]);
        }
        const float4 a4 = ldg4(A + o);
        a[0] = a4.x; a[1] = a4.y; a[2] = a4.z; a[3] = a4.w;
        if (B) {
            const float4 b4 = ldg4(B + o);
            b[0] = b4.x; b[1] = b4.y; b[2] = b4.z; b[3] = b4.w;
        }
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            if (4 * c + i >= W) {                          // row padding (may hold NaN): zero in the record,
                d[i] = 0.f;                                // never in the sums
                continue;
            }
            pc += (double)d[i] * (double)a[i];
            if (B) pb += (double)d[i] * (double)b[i];
        }
        *reinterpret_cast<float4*>(D + v * ldd + 4 * c) = make_float4(d[0], d[1], d[2], d[3]);
    }
    for (int off = lph >> 1; off; off >>= 1) {
        pc += __shfl_xor_sync(0xffffffffu, pc, off, LR);
        pb += __shfl_xor_sync(0xffffffffu, pb, off, LR);
    }
    if (!valid || (c % lph) != 0 || h >= H) return;
    const int64_t i = v * H + h;
    if (B) der[i] = (float)(pb - pc * (double)__ldg(bsum + i));
    float* aux = D + v * ldd + rec_aux_offset(W) + 4 * h;
    aux[0] = __ldg(er + i);
    const float l = __ldg(lse + i);
    aux[1] = l;
    aux[2] = (float)pc;
    aux[3] = -l * kLog2e;
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
#pragma unroll 4
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

// vectorised stage 1 for float4-aligned rows with W = H*F <= 128 (H == 1 or F % 4 == 0): LR = pow2(ceil(W/4)) lanes
// per row, 32/LR rows per warp instruction, two row groups in flight per warp; per-lane float4 partials of
// da_l / da_r merged in a fixed (warp, row-slot) order through shared memory.  Same outputs as stage 1 above.
template <int LR>
__global__ void __launch_bounds__(256) k_gat_attn_proj_bwd4(const float* __restrict__ T, int64_t M, int H, int F,
                                                            int64_t ldt, const float* __restrict__ a_l,
                                                            const float* __restrict__ a_r,
                                                            const float* __restrict__ del,
                                                            const float* __restrict__ der, float* __restrict__ dT,
                                                            int64_t rows_per_block, float* __restrict__ part) {
    constexpr int RPW = 32 / LR;
    __shared__ __align__(16) float red[8][RPW][2][4 * LR];
    const int W = H * F, C4 = (W + 3) / 4;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int c = lane % LR, sub = lane / LR;
    const bool act = c < C4;
    const int nv = act ? min(4, W - 4 * c) : 0;          // valid columns of this chunk (row padding past W)
    const int h = act ? (H == 1 ? 0 : (4 * c) / F) : 0;
    const int64_t r0 = blockIdx.x * rows_per_block;
    const int64_t r1 = min(M, r0 + rows_per_block);
    float4 al4 = make_float4(0.f, 0.f, 0.f, 0.f), ar4 = al4, sl = al4, sr = al4;
    if (act) {
        float* pa = &al4.x;
        float* pr = &ar4.x;
#pragma unroll
        for (int q = 0; q < 4; ++q)
            if (q < nv) { pa[q] = __ldg(a_l + 4 * c + q); pr[q] = __ldg(a_r + 4 * c + q); }
    }
    const int64_t stride = 8 * RPW;
    for (int64_t rb = r0 + w * RPW + sub; rb < r1; rb += 2 * stride) {
#pragma unroll
        for (int u = 0; u < 2; ++u) {
            const int64_t r = rb + u * stride;
            if (!act || r >= r1) continue;
            const float dl = del ? __ldg(del + r * H + h) : 0.f;
            const float dr = der ? __ldg(der + r * H + h) : 0.f;
            float4 t = ldg4(T + r * ldt + 4 * c);
            if (nv < 4) {                                    // padding columns: out of the sums, dT unchanged
                t.w = 0.f;
                if (nv < 3) t.z = 0.f;
                if (nv < 2) t.y = 0.f;
            }
            float4* pd = reinterpret_cast<float4*>(dT + r * ldt + 4 * c);
            float4 d = *pd;
            d.x += dl * al4.x + dr * ar4.x; d.y += dl * al4.y + dr * ar4.y;
            d.z += dl * al4.z + dr * ar4.z; d.w += dl * al4.w + dr * ar4.w;
            *pd = d;
            sl.x = fmaf(dl, t.x, sl.x); sl.y = fmaf(dl, t.y, sl.y); sl.z = fmaf(dl, t.z, sl.z); sl.w = fmaf(dl, t.w, sl.w);
            sr.x = fmaf(dr, t.x, sr.x); sr.y = fmaf(dr, t.y, sr.y); sr.z = fmaf(dr, t.z, sr.z); sr.w = fmaf(dr, t.w, sr.w);
        }
    }
    reinterpret_cast<float4*>(red[w][sub][0])[c] = sl;
    reinterpret_cast<float4*>(red[w][sub][1])[c] = sr;
    __syncthreads();
    float* pl = part + (int64_t)blockIdx.x * 2 * W;
    for (int i = threadIdx.x; i < 2 * W; i += blockDim.x) {
        const int which = i / W, j = i % W;
        float x = 0.f;
        for (int ww = 0; ww < 8; ++ww)
#pragma unroll
            for (int q = 0; q < RPW; ++q) x += red[ww][q][which][j];
        pl[which * W + j] = x;
    }
}

static int64_t proj_bwd_blocks(int64_t M) {
    int64_t b = 8 * num_sms();
    if (M < b * 64) b = (M + 63) / 64;
    return b < 1 ? 1 : b;
}

// ============================================================================================
// launch helpers
// ============================================================================================
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
    const int64_t ldel = el_stride(T, el, H, F, ldt);
    SS_ARG(ldel == H || ldt >= (int64_t)H * F + H, "gat_attn_proj: el packed into T needs ldt >= H*F + H");
    k_gat_attn_proj<<<(unsigned)((n + 255) / 256), 256, 0, to_stream(stream)>>>(T, M, H, F, ldt, a_l, a_r, el, er,
                                                                                ldel);
    return check_launch("k_gat_attn_proj");
}

seastar_status seastar_gat_fwd(seastar_graph g, const float* T_all, const float* el_all, const float* er_loc,
                               int32_t H, int32_t F, int64_t ldt, float slope, const float* bias, seastar_act act,
                               float* A_loc, float* Y_loc, float* lse_loc, float* B_loc, float* b_loc,
                               const seastar_dropout_spec* attn_drop, seastar_stream stream) {
    SS_ARG(g && T_all && el_all && er_loc && A_loc && Y_loc && lse_loc, "gat_fwd: NULL argument");
    SS_ARG((B_loc == nullptr) == (b_loc == nullptr), "gat_fwd: pass both B_loc and b_loc or neither");
    SS_ARG(!B_loc || (aligned16(B_loc) == aligned16(A_loc)), "gat_fwd: B_loc must be aligned like A_loc");
    SS_ARG(ldt < (int64_t(1) << 31), "gat_fwd: ldt must be < 2^31");
    SS_ARG(H >= 1 && F >= 1 && ldt >= (int64_t)H * F, "gat_fwd: bad sizes H=%d F=%d ldt=%lld", H, F, (long long)ldt);
    SS_ARG(act >= SEASTAR_ACT_NONE && act <= SEASTAR_ACT_SIGMOID, "gat_fwd: bad activation");
    SS_TRY(check_device());
    cudaStream_t s = to_stream(stream);
    GatFwdArgs a{};
    a.perm = g->fwd.perm; a.off = g->fwd.off; a.nbr = g->fwd.nbr;
    a.vbase = g->row_begin;
    a.T = T_all; a.el = el_all; a.er = er_loc;
    a.ldel = el_stride(T_all, el_all, H, F, ldt);
    SS_ARG(a.ldel == H || ldt >= (int64_t)H * F + H, "gat_fwd: el packed into T needs ldt >= H*F + H");
    a.H = H; a.F = F; a.ld = ldt; a.slope = slope; a.bias = bias; a.act = act;
    a.A = A_loc; a.Y = Y_loc; a.lse = lse_loc; a.B = B_loc; a.bsum = b_loc;
    a.row_begin = 0; a.row_end = g->fwd.n_rows;
    SS_ARG(!attn_drop || (attn_drop->p >= 0.f && attn_drop->p < 1.f), "gat_fwd: need 0 <= attn_drop->p < 1");
    set_drop(a, attn_drop, g->fwd.eid);
    if (!a.deid && launch_gat_fwd_hpl(a, long_rows(g->fwd), s)) return check_launch("k_gat_fwd_hpl");
    if (!a.deid && launch_gat_fwd_h1(a, long_rows(g->fwd), g->fwd.bucket_rows[1], g->fwd.pow2_rows[kH1MidClass], g->fwd.n_rows, s))
        return check_launch("k_gat_fwd_h1");
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
    const int W = H * F, C4 = (W + 3) / 4;
    const bool geo4 = W <= 128 && ldt % 4 == 0 && aligned16(dY_loc) && aligned16(A_loc) && aligned16(D_loc) &&
                      (!Y_loc || aligned16(Y_loc)) && (!B_loc || aligned16(B_loc)) &&
                      (H == 1 || (F % 4 == 0 && ((F / 4) & (F / 4 - 1)) == 0 && F / 4 <= 32));
    if (geo4) {
        const int LR = pow2_ceil(C4);
        const unsigned grid = (unsigned)((M * LR + 255) / 256);
        const int64_t ldd = seastar_gat_record_ld(H, F);
        cudaStream_t s = to_stream(stream);
#define PREP4(LRV) k_gat_bwd_prep4<LRV><<<grid, 256, 0, s>>>(M, H, F, ldt, dY_loc, Y_loc, act, A_loc, er_loc, lse_loc, \
                                                             D_loc, ldd, B_loc, b_loc, der_loc)
        switch (LR) {
            case 1: PREP4(1); break;
            case 2: PREP4(2); break;
            case 4: PREP4(4); break;
            case 8: PREP4(8); break;
            case 16: PREP4(16); break;
            default: PREP4(32); break;
        }
#undef PREP4
        return check_launch("k_gat_bwd_prep4");
    }
    SS_ARG(H <= 8 || (32 % F == 0 && H <= 32), "gat_bwd_prep: H > 8 needs F dividing 32 (and H <= 32)");
    k_gat_bwd_prep<<<(unsigned)((M + 7) / 8), 256, 0, to_stream(stream)>>>(
        M, H, F, ldt, dY_loc, Y_loc, act, A_loc, er_loc, lse_loc, D_loc, seastar_gat_record_ld(H, F), B_loc, b_loc,
        der_loc);
    return check_launch("k_gat_bwd_prep");
}

seastar_status seastar_gat_bwd(seastar_graph g, const float* T_loc, const float* el_loc, const float* D_all,
                               int32_t H, int32_t F, int64_t ldt, float slope, float* dT_loc, float* del_loc,
                               const seastar_dropout_spec* attn_drop, seastar_stream stream) {
    SS_ARG(g && T_loc && el_loc && D_all && dT_loc && del_loc, "gat_bwd: NULL argument");
    SS_ARG(ldt < (int64_t(1) << 31), "gat_bwd: ldt must be < 2^31");
    SS_ARG(H >= 1 && F >= 1 && ldt >= (int64_t)H * F, "gat_bwd: bad sizes");
    SS_TRY(check_device());
    cudaStream_t s = to_stream(stream);
    GatBwdArgs a{};
    a.perm = g->rev.perm; a.off = g->rev.off; a.nbr = g->rev.nbr;
    a.vbase = g->row_begin;
    a.T = T_loc; a.el = el_loc; a.D = D_all;
    a.ldel = el_stride(T_loc, el_loc, H, F, ldt);
    SS_ARG(a.ldel == H || ldt >= (int64_t)H * F + H, "gat_bwd: el packed into T needs ldt >= H*F + H");
    a.H = H; a.F = F; a.ldt = ldt; a.ldd = seastar_gat_record_ld(H, F); a.slope = slope;
    a.dT = dT_loc; a.del = del_loc;
    ScopedL2Window win(D_all, (size_t)g->N * a.ldd * sizeof(float));
    a.row_begin = 0; a.row_end = g->rev.n_rows;
    SS_ARG(!attn_drop || (attn_drop->p >= 0.f && attn_drop->p < 1.f), "gat_bwd: need 0 <= attn_drop->p < 1");
    set_drop(a, attn_drop, g->rev.eid);
    if (!a.deid && launch_gat_bwd_hpl(a, long_rows(g->rev), s)) return check_launch("k_gat_bwd_hpl");
    if (!a.deid && launch_gat_bwd_h1(a, long_rows(g->rev), g->rev.bucket_rows[1], g->rev.pow2_rows[kH1MidClass], g->rev.n_rows, false, s))
        return check_launch("k_gat_bwd_h1");
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
                               int32_t F, int64_t ldt, float slope, float* der_loc,
                               const seastar_dropout_spec* attn_drop, seastar_stream stream) {
    SS_ARG(g && T_all && el_all && D_loc && der_loc, "gat_der: NULL argument");
    SS_ARG(ldt < (int64_t(1) << 31), "gat_der: ldt must be < 2^31");
    SS_ARG(H >= 1 && F >= 1 && ldt >= (int64_t)H * F, "gat_der: bad sizes");
    SS_TRY(check_device());
    cudaStream_t s = to_stream(stream);
    GatBwdArgs a{};
    a.perm = g->fwd.perm; a.off = g->fwd.off; a.nbr = g->fwd.nbr;
    a.vbase = g->row_begin;
    a.T = T_all; a.el = el_all; a.D = D_loc;
    a.ldel = el_stride(T_all, el_all, H, F, ldt);
    SS_ARG(a.ldel == H || ldt >= (int64_t)H * F + H, "gat_der: el packed into T needs ldt >= H*F + H");
    a.H = H; a.F = F; a.ldt = ldt; a.ldd = seastar_gat_record_ld(H, F); a.slope = slope;
    a.der = der_loc;
    a.row_begin = 0; a.row_end = g->fwd.n_rows;
    SS_ARG(!attn_drop || (attn_drop->p >= 0.f && attn_drop->p < 1.f), "gat_der: need 0 <= attn_drop->p < 1");
    set_drop(a, attn_drop, g->fwd.eid);
    if (!a.deid && launch_gat_der_hpl(a, s)) return check_launch("k_gat_der_hpl");
    if (!a.deid && launch_gat_bwd_h1(a, long_rows(g->fwd), g->fwd.bucket_rows[1], g->fwd.pow2_rows[kH1MidClass], g->fwd.n_rows, true, s))
        return check_launch("k_gat_der_h1");
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
    const bool vec = W <= 128 && (H == 1 || F % 4 == 0) && ldt % 4 == 0 && aligned16(T) && aligned16(dT);
    if (vec) {
        const int LR = pow2_ceil((W + 3) / 4);
#define PROJ4(LRV) k_gat_attn_proj_bwd4<LRV><<<(unsigned)nblk, 256, 0, s>>>(T, M, H, F, ldt, a_l, a_r, del, der, dT, \
                                                                         rpb > 0 ? rpb : 1, part)
        switch (LR) {
            case 1: PROJ4(1); break;
            case 2: PROJ4(2); break;
            case 4: PROJ4(4); break;
            case 8: PROJ4(8); break;
            case 16: PROJ4(16); break;
            default: PROJ4(32); break;
        }
#undef PROJ4
    } else {
        k_gat_attn_proj_bwd1<<<(unsigned)nblk, 256, 0, s>>>(T, M, H, F, ldt, a_l, a_r, del, der, dT, rpb > 0 ? rpb : 1,
                                                            part);
    }
    reduce_splits(part, nblk, 2 * (int64_t)W, W, W, W, da_l, s);
    reduce_splits(part + W, nblk, 2 * (int64_t)W, W, W, W, da_r, s);
    return check_launch("k_gat_attn_proj_bwd");
}

}  // extern "C"
