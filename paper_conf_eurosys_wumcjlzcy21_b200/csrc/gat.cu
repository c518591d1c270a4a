// gat.cu -- a6 / a9: fused GAT layer (Fig. 2 L95-L123, Fig. 3 L159 src lines 9-23).
//
// Forward: the paper's FSM splits the GAT forward into 2 fused units at the Div (L391-L393:
// AggSum of exp, then Div -> Mul -> AggSum).  On B200 it is ONE pass over in(v): an online
// softmax keeps (running max m, running sum S, running weighted row acc) per head in registers, so
// no E-sized intermediate and no second gather of T are needed.  lse = m + log S is saved for the
// backward.
//
// Backward (§6.3.4: the Aggregation stage becomes the Source stage on the reverse CSR):
//   row pass (gat_bwd_prep): dA = dY act'(Y), c[v,h] = <dA[v,h], A[v,h]> (= sum_e a_e <dA_v, T_u>,
//     which removes the softmax-Jacobian pass), packed with er and lse into one record D[v];
//   source-major pass (gat_bwd): per u, per out-edge (u->v): a_e from lse, g_e = <dA_v, T_u> with
//     T_u held in registers, ds_e = a_e (g_e - c_v) LReLU'(s_e); dT_u += a_e dA_v and del_u += ds_e
//     accumulate in registers (no atomics); ds_e is stored at the edge's forward position;
//   der (gat_der): dst-major coalesced segment sum of ds over each forward row.
#include <math.h>

#include "common.cuh"

namespace seastar {

__device__ __forceinline__ float lrelu(float x, float slope) { return x > 0.f ? x : slope * x; }

struct GatFwdArgs {
    const int32_t* perm; const int32_t* off; const int32_t* nbr;
    int64_t row_begin, row_end, vbase;
    const float* T; const float* el; const float* er;
    int H, F; int64_t ld; float slope;
    const float* bias; int act;
    float* A; float* Y; float* lse;
};

// lane geometry shared by the GAT kernels: chunk `chunk` covers floats [chunk*VEC, chunk*VEC+VEC)
// of a row of W = H*F floats; with VEC = 4 every chunk lies inside one head (F % 4 == 0 or H == 1)
template <int VEC>
__device__ __forceinline__ int head_of(int chunk, int F, int H) {
    return H == 1 ? 0 : (chunk * VEC) / F;
}

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

    float m = -INFINITY, ssum = 0.f, acc[VEC];
#pragma unroll
    for (int i = 0; i < VEC; ++i) acc[i] = 0.f;

    for (int base = beg; base < end; base += RL) {
        const int n = min(RL, end - base);
        const int my = (gl < n) ? __ldg(a.nbr + base + gl) : 0;
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
#pragma unroll
            for (int i = 0; i < VEC; ++i) acc[i] *= corr;
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) {
                const float p = (z[jj] == -INFINITY) ? 0.f : expf(z[jj] - mb);
                ssum += p;
#pragma unroll
                for (int i = 0; i < VEC; ++i) acc[i] = fmaf(p, val[jj][i], acc[i]);
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
#pragma unroll
        for (int i = 0; i < VEC; ++i) acc[i] = acc[i] * ca + ao[i] * cb;
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
    if ((a.H == 1 && chunk == 0) || (a.H > 1 && col % a.F == 0))
        a.lse[v * a.H + h] = ssum > 0.f ? m + logf(ssum) : -INFINITY;
}

struct GatBwdArgs {
    const int32_t* perm; const int32_t* off; const int32_t* nbr; const int32_t* pos;
    int64_t row_begin, row_end, vbase;
    const float* T; const float* el; const float* D;
    int H, F; int64_t ldt, ldd; float slope;
    float* dT; float* del; float* ds;
};

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
    // lanes of head h inside the edge group: [hs, hs + lph)
    const int lph = (a.H == 1) ? C : (a.F / VEC);
    const int hc = active ? (a.H == 1 ? chunk : chunk - h * lph) : 0;
    const int hs = c - hc;

    float t[VEC];
    if (valid && active) load_vec<VEC>(a.T + u * a.ldt + col, t);
#pragma unroll
    for (int i = 0; i < VEC; ++i)   // padding columns never enter the head dot products
        if (!(valid && active) || col + i >= W) t[i] = 0.f;
    const float elu = (valid && active) ? __ldg(a.el + u * a.H + h) : 0.f;
    float acc[VEC], dl = 0.f;
#pragma unroll
    for (int i = 0; i < VEC; ++i) acc[i] = 0.f;

    for (int base = beg; base < end; base += RL) {
        const int n = min(RL, end - base);
        const int myv = (gl < n) ? __ldg(a.nbr + base + gl) : 0;
        const int myp = (gl < n) ? __ldg(a.pos + base + gl) : 0;
#pragma unroll
        for (int j0 = 0; j0 < L; j0 += UB) {
            if (j0 * S >= n) break;
            float dA[UB][VEC], er[UB], lse[UB], cv[UB];
            int pe[UB];
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) {
                const int k = (j0 + jj) * S + slot;
                const int v = __shfl_sync(gmask, myv, k & (RL - 1), RL);
                pe[jj] = __shfl_sync(gmask, myp, k & (RL - 1), RL);
                if (k < n && active) {
                    const float* rec = a.D + (int64_t)v * a.ldd;
                    load_vec<VEC>(rec + col, dA[jj]);
#pragma unroll
                    for (int i = 0; i < VEC; ++i)
                        if (col + i >= W) dA[jj][i] = 0.f;
                    const float* aux = rec + ((W + 3) & ~3) + 4 * h;
                    if constexpr (VEC == 4) {
                        if ((a.ldd & 3) == 0) {
                            const float4 x = ldg4(aux);
                            er[jj] = x.x; lse[jj] = x.y; cv[jj] = x.z;
                        } else {
                            er[jj] = __ldg(aux); lse[jj] = __ldg(aux + 1); cv[jj] = __ldg(aux + 2);
                        }
                    } else {
                        er[jj] = __ldg(aux); lse[jj] = __ldg(aux + 1); cv[jj] = __ldg(aux + 2);
                    }
                } else {
#pragma unroll
                    for (int i = 0; i < VEC; ++i) dA[jj][i] = 0.f;
                    er[jj] = 0.f; lse[jj] = INFINITY; cv[jj] = 0.f;
                }
            }
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) {
                const int k = (j0 + jj) * S + slot;
                // g = <dA_v[h], T_u[h]> : segmented reduction over the lanes of head h, then broadcast
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
                    const float ds = al * (g - cv[jj]) * (s > 0.f ? 1.f : a.slope);
#pragma unroll
                    for (int i = 0; i < VEC; ++i) acc[i] = fmaf(al, dA[jj][i], acc[i]);
                    dl += ds;
                    if (hc == 0) a.ds[(int64_t)pe[jj] * a.H + h] = ds;
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

// der[v,h] = sum over row of ds[j*H + h]; warp per row, rows given by (perm or identity, off)
__global__ void __launch_bounds__(256) k_gat_der(const int32_t* __restrict__ perm, const int32_t* __restrict__ off,
                                                 int64_t n_rows, int64_t vbase, const float* __restrict__ ds, int H,
                                                 float* __restrict__ der) {
    const int lane = threadIdx.x & 31;
    const int64_t row = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    if (row >= n_rows) return;
    const int64_t beg = (int64_t)__ldg(off + row) * H, end = (int64_t)__ldg(off + row + 1) * H;
    const int64_t v = (perm ? (int64_t)__ldg(perm + row) : row) - vbase;
    if ((32 % H) == 0) {
        float x0 = 0.f, x1 = 0.f;
        int64_t i = beg + lane;
        for (; i + 32 < end; i += 64) {   // two loads in flight
            x0 += __ldg(ds + i);
            x1 += __ldg(ds + i + 32);
        }
        if (i < end) x0 += __ldg(ds + i);
        float x = x0 + x1;
        // lanes l and l' share a head iff l = l' (mod H); the row block starts at a multiple of H
        for (int o = H; o < 32; o <<= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
        if (lane < H) der[v * H + lane] = x;
    } else {
        for (int hh = lane; hh < H; hh += 32) {
            float x = 0.f;
            for (int64_t i = beg + hh; i < end; i += H) x += __ldg(ds + i);
            der[v * H + hh] = x;
        }
    }
}

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
                               int64_t ldd) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i >= M * H) return;
    const int64_t v = i / H;
    const int h = (int)(i % H);
    const int64_t o = v * ldt + (int64_t)h * F;
    float* rec = D + v * ldd;
    float cdot = 0.f;
    for (int f = 0; f < F; ++f) {
        float d = __ldg(dY + o + f);
        if (act != SEASTAR_ACT_NONE) d *= act_grad_from_y(act, __ldg(Y + o + f));
        rec[(int64_t)h * F + f] = d;
        cdot = fmaf(d, __ldg(A + o + f), cdot);
    }
    float* aux = rec + (((int64_t)H * F + 3) & ~3LL) + 4 * h;
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

template <int VEC, int L>
static void gat_fwd_launch(GatFwdArgs a, int64_t split, int64_t n_rows, cudaStream_t s) {
    GatFwdArgs hi = a, lo = a;
    hi.row_begin = 0; hi.row_end = split;
    lo.row_begin = split; lo.row_end = n_rows;
    if (split > 0) k_gat_fwd<VEC, L, 32><<<(unsigned)((split + 7) / 8), 256, 0, s>>>(hi);
    if (n_rows > split) {
        constexpr int RL = L < 4 ? 4 : L;
        const int64_t per = 256 / RL;
        k_gat_fwd<VEC, L, RL><<<(unsigned)((n_rows - split + per - 1) / per), 256, 0, s>>>(lo);
    }
}
template <int VEC, int L>
static void gat_bwd_launch(GatBwdArgs a, int64_t split, int64_t n_rows, cudaStream_t s) {
    GatBwdArgs hi = a, lo = a;
    hi.row_begin = 0; hi.row_end = split;
    lo.row_begin = split; lo.row_end = n_rows;
    if (split > 0) k_gat_bwd<VEC, L, 32><<<(unsigned)((split + 7) / 8), 256, 0, s>>>(hi);
    if (n_rows > split) {
        constexpr int RL = L < 4 ? 4 : L;
        const int64_t per = 256 / RL;
        k_gat_bwd<VEC, L, RL><<<(unsigned)((n_rows - split + per - 1) / per), 256, 0, s>>>(lo);
    }
}

}  // namespace seastar

using namespace seastar;

#define GAT_DISPATCH(FN, VEC, L, ...)          \
    switch (L) {                               \
        case 1: FN<VEC, 1>(__VA_ARGS__); break;  \
        case 2: FN<VEC, 2>(__VA_ARGS__); break;  \
        case 4: FN<VEC, 4>(__VA_ARGS__); break;  \
        case 8: FN<VEC, 8>(__VA_ARGS__); break;  \
        case 16: FN<VEC, 16>(__VA_ARGS__); break; \
        default: FN<VEC, 32>(__VA_ARGS__); break; \
    }

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
                               float* A_loc, float* Y_loc, float* lse_loc, seastar_stream stream) {
    SS_ARG(g && T_all && el_all && er_loc && A_loc && Y_loc && lse_loc, "gat_fwd: NULL argument");
    SS_ARG(H >= 1 && F >= 1 && ldt >= (int64_t)H * F, "gat_fwd: bad sizes H=%d F=%d ldt=%lld", H, F, (long long)ldt);
    SS_ARG(act >= SEASTAR_ACT_NONE && act <= SEASTAR_ACT_SIGMOID, "gat_fwd: bad activation");
    SS_TRY(check_device());
    const bool vec4 = (ldt % 4 == 0) && (H == 1 || F % 4 == 0) && aligned16(T_all) && aligned16(A_loc) &&
                      aligned16(Y_loc);
    const int VEC = vec4 ? 4 : 1;
    const int C = (H * F + VEC - 1) / VEC;
    SS_ARG(C <= 32, "gat_fwd: row of H*F=%d floats exceeds 32 lanes x %d", H * F, VEC);
    const int L = pow2_ceil(C);
    GatFwdArgs a{};
    a.perm = g->fwd.perm; a.off = g->fwd.off; a.nbr = g->fwd.nbr;
    a.vbase = g->row_begin;
    a.T = T_all; a.el = el_all; a.er = er_loc;
    a.H = H; a.F = F; a.ld = ldt; a.slope = slope; a.bias = bias; a.act = act;
    a.A = A_loc; a.Y = Y_loc; a.lse = lse_loc;
    const int64_t split = L >= 32 ? g->fwd.n_rows : g->fwd.bucket_rows[1];
    cudaStream_t s = to_stream(stream);
    if (vec4) { GAT_DISPATCH(gat_fwd_launch, 4, L, a, split, g->fwd.n_rows, s); }
    else { GAT_DISPATCH(gat_fwd_launch, 1, L, a, split, g->fwd.n_rows, s); }
    return check_launch("k_gat_fwd");
}

seastar_status seastar_gat_bwd_prep(seastar_graph g, const float* dY_loc, const float* Y_loc, seastar_act act,
                                    const float* A_loc, const float* er_loc, const float* lse_loc, int32_t H,
                                    int32_t F, int64_t ldt, float* D_loc, seastar_stream stream) {
    SS_ARG(g && dY_loc && A_loc && er_loc && lse_loc && D_loc, "gat_bwd_prep: NULL argument");
    SS_ARG(act == SEASTAR_ACT_NONE || Y_loc, "gat_bwd_prep: Y_loc is required for act != NONE");
    SS_ARG(H >= 1 && F >= 1 && ldt >= (int64_t)H * F, "gat_bwd_prep: bad sizes");
    SS_TRY(check_device());
    const int64_t M = g->n_loc();
    if (M == 0) return SEASTAR_OK;
    const int64_t n = M * H;
    k_gat_bwd_prep<<<(unsigned)((n + 255) / 256), 256, 0, to_stream(stream)>>>(
        M, H, F, ldt, dY_loc, Y_loc, act, A_loc, er_loc, lse_loc, D_loc, seastar_gat_record_ld(H, F));
    return check_launch("k_gat_bwd_prep");
}

seastar_status seastar_gat_bwd(seastar_graph g, const float* T_loc, const float* el_loc, const float* D_all,
                               int32_t H, int32_t F, int64_t ldt, float slope, float* dT_loc, float* del_loc,
                               float* ds_work, seastar_stream stream) {
    SS_ARG(g && T_loc && el_loc && D_all && dT_loc && del_loc && ds_work, "gat_bwd: NULL argument");
    SS_ARG(H >= 1 && F >= 1 && ldt >= (int64_t)H * F, "gat_bwd: bad sizes");
    SS_TRY(check_device());
    const int64_t ldd = seastar_gat_record_ld(H, F);
    const bool vec4 = (ldt % 4 == 0) && (H == 1 || F % 4 == 0) && aligned16(T_loc) && aligned16(D_all) &&
                      aligned16(dT_loc);
    const int VEC = vec4 ? 4 : 1;
    const int C = (H * F + VEC - 1) / VEC;
    SS_ARG(C <= 32, "gat_bwd: row of H*F=%d floats exceeds 32 lanes x %d", H * F, VEC);
    const int L = pow2_ceil(C);
    GatBwdArgs a{};
    a.perm = g->rev.perm; a.off = g->rev.off; a.nbr = g->rev.nbr; a.pos = g->rev.pos;
    a.vbase = g->row_begin;
    a.T = T_loc; a.el = el_loc; a.D = D_all;
    a.H = H; a.F = F; a.ldt = ldt; a.ldd = ldd; a.slope = slope;
    a.dT = dT_loc; a.del = del_loc; a.ds = ds_work;
    const int64_t split = L >= 32 ? g->rev.n_rows : g->rev.bucket_rows[1];
    cudaStream_t s = to_stream(stream);
    if (vec4) { GAT_DISPATCH(gat_bwd_launch, 4, L, a, split, g->rev.n_rows, s); }
    else { GAT_DISPATCH(gat_bwd_launch, 1, L, a, split, g->rev.n_rows, s); }
    return check_launch("k_gat_bwd");
}

seastar_status seastar_gat_der(seastar_graph g, const float* ds_work, int32_t H, float* der, seastar_stream stream) {
    SS_ARG(g && ds_work && der, "gat_der: NULL argument");
    SS_ARG(H >= 1, "gat_der: bad H");
    SS_TRY(check_device());
    cudaStream_t s = to_stream(stream);
    if (!g->partitioned) {
        const int64_t n = g->fwd.n_rows;
        if (n) k_gat_der<<<(unsigned)((n + 7) / 8), 256, 0, s>>>(g->fwd.perm, g->fwd.off, n, g->row_begin, ds_work, H, der);
    } else {
        const int64_t n = g->lsf.n_rows;
        if (n) k_gat_der<<<(unsigned)((n + 7) / 8), 256, 0, s>>>(nullptr, g->lsf.off, n, 0, ds_work, H, der);
    }
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
