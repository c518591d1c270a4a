// gat_hpl.cu -- head-per-lane GAT edge kernels (H | 32, F % 4 == 0, F <= 32): a warp owns one row,
// lane = (edge slot, head) with S = 32 / H slots, each lane holds a whole head row of F floats so
// the per-(edge, head) softmax weight and the head dot products never leave the lane.
// PAPER.md Fig. 2 L95-L123 (GAT forward), Fig. 3 L159 src lines 9-23, §6.3.4 L461-L463 (the
// Aggregation stage of the backward runs on the reverse CSR).
//
// The inner loops are branch-free: H and F are template parameters, an out-of-range edge slot
// gathers row 0 (always valid memory) and gets weight 0, softmax weights are ex2 of one FFMA, and
// neighbour ids are software-pipelined one 32-edge chunk ahead (see gcn.cu).
#include <algorithm>

#include "gat_common.cuh"

namespace seastar {

// edges per lane per batch: as many as fit the 3-blocks/SM register budget
#ifndef GAT_HPL_FWD_UBMAX
#define GAT_HPL_FWD_UBMAX 4
#endif
template <int F4>
constexpr int hpl_ub() { return (F4 <= 2 ? 4 : (F4 <= 4 ? 2 : 1)) < GAT_HPL_FWD_UBMAX ? (F4 <= 2 ? 4 : (F4 <= 4 ? 2 : 1)) : GAT_HPL_FWD_UBMAX; }
#ifndef GAT_HPL_BWD_UBMAX
#define GAT_HPL_BWD_UBMAX 2   // measured: 4 spills at 80 regs and is 30% slower on Reddit (H=8, F=8)
#endif
template <int F4>
constexpr int hpl_bwd_ub() { return hpl_ub<F4>() < GAT_HPL_BWD_UBMAX ? hpl_ub<F4>() : GAT_HPL_BWD_UBMAX; }

// forward (FWD CSR, row = destination v).  Online softmax per (v, h): running max m, sum ssum,
// weighted row acc.  SB: also P_v = sum_{s_e > 0} a_e T_u, from which the epilogue writes the der
// factors B_v = sum_e a_e LReLU'(s_e) T_u and b_v = sum_e a_e LReLU'(s_e) (gat.cu, gat_bwd_prep).
#ifndef GAT_MB_FWD_HPL
#define GAT_MB_FWD_HPL GAT_MB_FWD
#endif
// WPR > 1 (WPR = the block's warps): the launch's first a.nlong blocks each own one long row (long_rows()), warp w
// runs the online softmax over the w-th contiguous slice of the row's edges, and the warps' (max, sum, weighted
// rows) are merged in warp order through shared memory by the same online-softmax merge as the slot tree
// (deterministic; "CTA + Warp"); every later block owns 8 rows, a warp each.
template <int H, int F4, bool SB, int WPR = 1>
__global__ void __launch_bounds__(256, GAT_MB_FWD_HPL) k_gat_fwd_hpl(const GatFwdArgs a) {
    constexpr int F = 4 * F4, S = 32 / H;
    constexpr int UE = hpl_ub<F4>() < H ? hpl_ub<F4>() : H;   // edges per lane per batch
    constexpr int NB = H / UE;                                // batches per 32-edge chunk
    const int lane = threadIdx.x & 31;
    const int h = lane % H, slot = lane / H;
    const int wib = threadIdx.x >> 5;
    const bool hubblk = WPR > 1 && (int64_t)blockIdx.x < a.nlong;      // block-uniform
    const int64_t row = hubblk ? a.row_begin + blockIdx.x
                      : WPR > 1 ? a.row_begin + a.nlong + ((int64_t)blockIdx.x - a.nlong) * (blockDim.x >> 5) + wib
                                : a.row_begin + ((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5);
    if (row >= a.row_end) return;                      // warp-uniform (never taken in a long-row block)
    int beg = __ldg(a.off + row), end = __ldg(a.off + row + 1);
    if (hubblk) {
        const int64_t len = end - beg;
        const int b0 = beg + (int)(len * wib / WPR);
        end = beg + (int)(len * (wib + 1) / WPR);
        beg = b0;
    }
    const int64_t v = (int64_t)__ldg(a.perm + row) - a.vbase;
    const float erv = __ldg(a.er + v * H + h);
    const float slope = a.slope;
    const float* Th = a.T + h * F;
    const float* elh = a.el + h;
    float m = kNegBig, mlog = kNegBig * kLog2e, ssum = 0.f, psum = 0.f;
    float acc[F], pacc[SB ? F : 1];
#pragma unroll
    for (int i = 0; i < F; ++i) acc[i] = 0.f;
#pragma unroll
    for (int i = 0; i < (SB ? F : 1); ++i) pacc[i] = 0.f;
    int nxt = (lane < end - beg) ? __ldcs(a.nbr + beg + lane) : 0;
    for (int base = beg; base < end; base += 32) {
        const int n = min(32, end - base);
        const int my = nxt;
        nxt = (lane < end - base - 32) ? __ldcs(a.nbr + base + 32 + lane) : 0;
#pragma unroll
        for (int b = 0; b < NB; ++b) {
            if (b * UE * S >= n) break;                    // warp-uniform
            float z[UE];
            float4 x[UE][F4];
#pragma unroll
            for (int jj = 0; jj < UE; ++jj) {
                const int k = slot + S * (b * UE + jj);    // < 32
                const int u = __shfl_sync(0xffffffffu, my, k);   // 0 for k >= n: a valid row
                const float* tp = row_ptr(Th, u, a.ld);
#pragma unroll
                for (int q = 0; q < F4; ++q) x[jj][q] = ldg4(tp + 4 * q);
                const float s = __ldg(elh + (size_t)(uint32_t)u * H) + erv;
                z[jj] = k < n ? lrelu(s, slope) : -INFINITY;
            }
            float mb = m;
#pragma unroll
            for (int jj = 0; jj < UE; ++jj) mb = fmaxf(mb, z[jj]);
            if (mb > m) {                                  // rescale only when the running max moves
                const float corr = ex2((m - mb) * kLog2e);
                ssum *= corr;
#pragma unroll
                for (int i = 0; i < F; ++i) acc[i] *= corr;
                if (SB) {
                    psum *= corr;
#pragma unroll
                    for (int i = 0; i < (SB ? F : 1); ++i) pacc[i] *= corr;
                }
                m = mb;
                mlog = mb * kLog2e;
            }
#pragma unroll
            for (int jj = 0; jj < UE; ++jj) {
                const float p = ex2(fmaf(z[jj], kLog2e, -mlog));   // 0 for an empty slot
                ssum += p;
#pragma unroll
                for (int q = 0; q < F4; ++q) {
                    acc[4 * q] = fmaf(p, x[jj][q].x, acc[4 * q]);
                    acc[4 * q + 1] = fmaf(p, x[jj][q].y, acc[4 * q + 1]);
                    acc[4 * q + 2] = fmaf(p, x[jj][q].z, acc[4 * q + 2]);
                    acc[4 * q + 3] = fmaf(p, x[jj][q].w, acc[4 * q + 3]);
                }
                if (SB) {
                    const float pp = z[jj] > 0.f ? p : 0.f;
                    psum += pp;
#pragma unroll
                    for (int q = 0; q < (SB ? F4 : 0); ++q) {
                        pacc[(4 * q) % (SB ? F : 1)] = fmaf(pp, x[jj][q].x, pacc[(4 * q) % (SB ? F : 1)]);
                        pacc[(4 * q + 1) % (SB ? F : 1)] = fmaf(pp, x[jj][q].y, pacc[(4 * q + 1) % (SB ? F : 1)]);
                        pacc[(4 * q + 2) % (SB ? F : 1)] = fmaf(pp, x[jj][q].z, pacc[(4 * q + 2) % (SB ? F : 1)]);
                        pacc[(4 * q + 3) % (SB ? F : 1)] = fmaf(pp, x[jj][q].w, pacc[(4 * q + 3) % (SB ? F : 1)]);
                    }
                }
            }
        }
    }
    // merge the S slots of each head (fixed xor tree: deterministic)
#pragma unroll
    for (int o = H; o < 32; o <<= 1) {
        const float mo = __shfl_xor_sync(0xffffffffu, m, o);
        const float so = __shfl_xor_sync(0xffffffffu, ssum, o);
        const float mn = fmaxf(m, mo);
        const float ca = ex2((m - mn) * kLog2e), cb = ex2((mo - mn) * kLog2e);
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
    if (hubblk) {                                      // merge the warps' slices in warp order, one warp at a time
        constexpr int NS = 3 + F + (SB ? F : 0);
        __shared__ float st[H][NS];
        for (int w2 = 1; w2 < WPR; ++w2) {
            if (wib == w2 && slot == 0) {
                float* p = st[h];
                p[0] = m; p[1] = ssum; p[2] = psum;
#pragma unroll
                for (int i = 0; i < F; ++i) p[3 + i] = acc[i];
#pragma unroll
                for (int i = 0; i < (SB ? F : 0); ++i) p[3 + F + i] = pacc[i % (SB ? F : 1)];
            }
            __syncthreads();
            if (wib == 0 && slot == 0) {
                const float* p = st[h];
                const float mo = p[0], mn = fmaxf(m, mo);
                const float ca = ex2((m - mn) * kLog2e), cb = ex2((mo - mn) * kLog2e);
                ssum = ssum * ca + p[1] * cb;
#pragma unroll
                for (int i = 0; i < F; ++i) acc[i] = acc[i] * ca + p[3 + i] * cb;
                if (SB) {
                    psum = psum * ca + p[2] * cb;
#pragma unroll
                    for (int i = 0; i < (SB ? F : 1); ++i) pacc[i] = pacc[i] * ca + p[3 + F + i] * cb;
                }
                m = mn;
            }
            __syncthreads();
        }
        if (wib != 0) return;
    }
    if (slot != 0) return;
    const float inv = ssum > 0.f ? 1.f / ssum : 0.f;
    const int64_t hoff = (int64_t)h * F;
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
            for (int i = 0; i < 4; ++i) b4[i] = slope * o4[i] + (1.f - slope) * pacc[(4 * q + i) % (SB ? F : 1)] * inv;
            *reinterpret_cast<float4*>(a.B + v * a.ld + hoff + 4 * q) = make_float4(b4[0], b4[1], b4[2], b4[3]);
        }
    }
    a.lse[v * H + h] = ssum > 0.f ? m + logf(ssum) : -INFINITY;
    if (SB) a.bsum[v * H + h] = ssum > 0.f ? slope + (1.f - slope) * psum * inv : 0.f;
}

// source-major backward (REV CSR, row = source u, out-edges u -> v; gathers the records D[v]):
//   a_e = exp(LReLU(s_e) - lse_v), g_e = <dA_v, T_u>, ds_e = a_e (g_e - c_v) LReLU'(s_e);
//   dT_u = sum_e a_e dA_v, del_u = sum_e ds_e  (registers only, no atomics)
// measured on Reddit (H = 8, F = 8): 4 resident blocks (64 registers, 16 bytes of spill) hide the record-gather
// latency of the source-major backward better than 3 (80 registers): 3.12 -> 2.64 ms; the forward loses at 4
#ifndef GAT_MB_BWD_HPL
#define GAT_MB_BWD_HPL 4
#endif
template <int H, int F4, int WPR = 1>
__global__ void __launch_bounds__(256, GAT_MB_BWD_HPL) k_gat_bwd_hpl(const GatBwdArgs a) {
    constexpr int F = 4 * F4, S = 32 / H;
    constexpr int UE = hpl_bwd_ub<F4>() < H ? hpl_bwd_ub<F4>() : H;
    constexpr int NB = H / UE;
    const int lane = threadIdx.x & 31;
    const int h = lane % H, slot = lane / H;
    const int wib = threadIdx.x >> 5;
    const bool hubblk = WPR > 1 && (int64_t)blockIdx.x < a.nlong;      // block-uniform
    const int64_t row = hubblk ? a.row_begin + blockIdx.x
                      : WPR > 1 ? a.row_begin + a.nlong + ((int64_t)blockIdx.x - a.nlong) * (blockDim.x >> 5) + wib
                                : a.row_begin + ((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5);
    if (row >= a.row_end) return;
    int beg = __ldg(a.off + row), end = __ldg(a.off + row + 1);
    if (hubblk) {                                      // long rows: warp w takes the w-th slice (see the forward)
        const int64_t len = end - beg;
        const int b0 = beg + (int)(len * wib / WPR);
        end = beg + (int)(len * (wib + 1) / WPR);
        beg = b0;
    }
    const int64_t u = (int64_t)__ldg(a.perm + row) - a.vbase;
    const int64_t hoff = (int64_t)h * F;
    const float slope = a.slope;
    float4 t[F4];
#pragma unroll
    for (int q = 0; q < F4; ++q) t[q] = ldg4(a.T + u * a.ldt + hoff + 4 * q);
    const float elu = __ldg(a.el + u * H + h);
    const float* Dh = a.D + hoff;
    const float* Xh = a.D + rec_aux_offset(H * F) + 4 * h;
    float acc[F], dl = 0.f;
#pragma unroll
    for (int i = 0; i < F; ++i) acc[i] = 0.f;
    int nxt = (lane < end - beg) ? __ldcs(a.nbr + beg + lane) : 0;
    for (int base = beg; base < end; base += 32) {
        const int n = min(32, end - base);
        const int my = nxt;
        nxt = (lane < end - base - 32) ? __ldcs(a.nbr + base + 32 + lane) : 0;
#pragma unroll
        for (int b = 0; b < NB; ++b) {
            if (b * UE * S >= n) break;
            float4 d[UE][F4], ax[UE];
            int kk[UE];
#pragma unroll
            for (int jj = 0; jj < UE; ++jj) {
                kk[jj] = slot + S * (b * UE + jj);
                const int v = __shfl_sync(0xffffffffu, my, kk[jj]);
                const float* rp = row_ptr(Dh, v, a.ldd);
#pragma unroll
                for (int q = 0; q < F4; ++q) d[jj][q] = ldg4(rp + 4 * q);
                ax[jj] = ldg4(row_ptr(Xh, v, a.ldd));      // (er, lse, c, nl2) of head h
            }
#pragma unroll
            for (int jj = 0; jj < UE; ++jj) {
                float g = 0.f;
#pragma unroll
                for (int q = 0; q < F4; ++q) {
                    g = fmaf(d[jj][q].x, t[q].x, g);
                    g = fmaf(d[jj][q].y, t[q].y, g);
                    g = fmaf(d[jj][q].z, t[q].z, g);
                    g = fmaf(d[jj][q].w, t[q].w, g);
                }
                const float s = elu + ax[jj].x;
                const bool pos = s > 0.f;
                const float al0 = ex2(fmaf(pos ? s : slope * s, kLog2e, ax[jj].w));
                const float al = kk[jj] < n ? al0 : 0.f;
                dl = fmaf(al * (g - ax[jj].z), pos ? 1.f : slope, dl);
#pragma unroll
                for (int q = 0; q < F4; ++q) {
                    acc[4 * q] = fmaf(al, d[jj][q].x, acc[4 * q]);
                    acc[4 * q + 1] = fmaf(al, d[jj][q].y, acc[4 * q + 1]);
                    acc[4 * q + 2] = fmaf(al, d[jj][q].z, acc[4 * q + 2]);
                    acc[4 * q + 3] = fmaf(al, d[jj][q].w, acc[4 * q + 3]);
                }
            }
        }
    }
#pragma unroll
    for (int o = H; o < 32; o <<= 1) {
#pragma unroll
        for (int i = 0; i < F; ++i) acc[i] += __shfl_xor_sync(0xffffffffu, acc[i], o);
        dl += __shfl_xor_sync(0xffffffffu, dl, o);
    }
    if (hubblk) {                                      // add the warps' slices in warp order, one warp at a time
        __shared__ float st[H][F + 1];
        for (int w2 = 1; w2 < WPR; ++w2) {
            if (wib == w2 && slot == 0) {
#pragma unroll
                for (int i = 0; i < F; ++i) st[h][i] = acc[i];
                st[h][F] = dl;
            }
            __syncthreads();
            if (wib == 0 && slot == 0) {
#pragma unroll
                for (int i = 0; i < F; ++i) acc[i] += st[h][i];
                dl += st[h][F];
            }
            __syncthreads();
        }
        if (wib != 0) return;
    }
    if (slot != 0) return;
    float* pd = a.dT + u * a.ldt + hoff;
#pragma unroll
    for (int q = 0; q < F4; ++q)
        *reinterpret_cast<float4*>(pd + 4 * q) = make_float4(acc[4 * q], acc[4 * q + 1], acc[4 * q + 2], acc[4 * q + 3]);
    a.del[u * H + h] = dl;
}

// destination-major der pass (FWD CSR, row = v): der_v = sum_{e in in(v)} ds_e, recomputing ds_e
// from the gathered T_u / el_u and v's own record (used when the forward did not save B / b)
template <int H, int F4>
__global__ void __launch_bounds__(256, GAT_MB_BWD) k_gat_der_hpl(const GatBwdArgs a) {
    constexpr int F = 4 * F4, S = 32 / H;
    constexpr int UE = hpl_ub<F4>() < H ? hpl_ub<F4>() : H;
    constexpr int NB = H / UE;
    const int lane = threadIdx.x & 31;
    const int h = lane % H, slot = lane / H;
    const int64_t row = a.row_begin + ((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5);
    if (row >= a.row_end) return;
    const int beg = __ldg(a.off + row), end = __ldg(a.off + row + 1);
    const int64_t v = (int64_t)__ldg(a.perm + row) - a.vbase;
    const int64_t hoff = (int64_t)h * F;
    const float slope = a.slope;
    const float* rec = a.D + v * a.ldd;
    float4 d[F4];
#pragma unroll
    for (int q = 0; q < F4; ++q) d[q] = ldg4(rec + hoff + 4 * q);
    const float4 ax = ldg4(rec + rec_aux_offset(H * F) + 4 * h);   // (er, lse, c, nl2)
    const float* Th = a.T + hoff;
    const float* elh = a.el + h;
    float dr = 0.f;
    int nxt = (lane < end - beg) ? __ldcs(a.nbr + beg + lane) : 0;
    for (int base = beg; base < end; base += 32) {
        const int n = min(32, end - base);
        const int my = nxt;
        nxt = (lane < end - base - 32) ? __ldcs(a.nbr + base + 32 + lane) : 0;
#pragma unroll
        for (int b = 0; b < NB; ++b) {
            if (b * UE * S >= n) break;
            float4 t[UE][F4];
            float el[UE];
            int kk[UE];
#pragma unroll
            for (int jj = 0; jj < UE; ++jj) {
                kk[jj] = slot + S * (b * UE + jj);
                const int u = __shfl_sync(0xffffffffu, my, kk[jj]);
                const float* tp = row_ptr(Th, u, a.ldt);
#pragma unroll
                for (int q = 0; q < F4; ++q) t[jj][q] = ldg4(tp + 4 * q);
                el[jj] = __ldg(elh + (size_t)(uint32_t)u * H);
            }
#pragma unroll
            for (int jj = 0; jj < UE; ++jj) {
                float g = 0.f;
#pragma unroll
                for (int q = 0; q < F4; ++q) {
                    g = fmaf(d[q].x, t[jj][q].x, g);
                    g = fmaf(d[q].y, t[jj][q].y, g);
                    g = fmaf(d[q].z, t[jj][q].z, g);
                    g = fmaf(d[q].w, t[jj][q].w, g);
                }
                const float s = el[jj] + ax.x;
                const bool pos = s > 0.f;
                const float al0 = ex2(fmaf(pos ? s : slope * s, kLog2e, ax.w));
                const float al = kk[jj] < n ? al0 : 0.f;
                dr = fmaf(al * (g - ax.z), pos ? 1.f : slope, dr);
            }
        }
    }
#pragma unroll
    for (int o = H; o < 32; o <<= 1) dr += __shfl_xor_sync(0xffffffffu, dr, o);
    if (slot == 0) a.der[v * H + h] = dr;
}

// ---------------------------------------------------------------------------------------------
// launchers: one warp per row over the whole index set
// ---------------------------------------------------------------------------------------------
#define SS_HPL_F4(KERNEL, H, f4, ...)                                                          \
    switch (f4) {                                                                              \
        case 1: launch_k(KERNEL<H, 1 __VA_ARGS__>, dim3(grid), dim3(256), 0, s, a); break;     \
        case 2: launch_k(KERNEL<H, 2 __VA_ARGS__>, dim3(grid), dim3(256), 0, s, a); break;     \
        case 3: launch_k(KERNEL<H, 3 __VA_ARGS__>, dim3(grid), dim3(256), 0, s, a); break;     \
        case 4: launch_k(KERNEL<H, 4 __VA_ARGS__>, dim3(grid), dim3(256), 0, s, a); break;     \
        case 5: launch_k(KERNEL<H, 5 __VA_ARGS__>, dim3(grid), dim3(256), 0, s, a); break;     \
        case 6: launch_k(KERNEL<H, 6 __VA_ARGS__>, dim3(grid), dim3(256), 0, s, a); break;     \
        case 7: launch_k(KERNEL<H, 7 __VA_ARGS__>, dim3(grid), dim3(256), 0, s, a); break;     \
        default: launch_k(KERNEL<H, 8 __VA_ARGS__>, dim3(grid), dim3(256), 0, s, a); break;    \
    }
#define SS_HPL_H(KERNEL, H, f4, ...)                                \
    switch (H) {                                                    \
        case 2: SS_HPL_F4(KERNEL, 2, f4, __VA_ARGS__) break;        \
        case 4: SS_HPL_F4(KERNEL, 4, f4, __VA_ARGS__) break;        \
        case 8: SS_HPL_F4(KERNEL, 8, f4, __VA_ARGS__) break;        \
        case 16: SS_HPL_F4(KERNEL, 16, f4, __VA_ARGS__) break;      \
        default: SS_HPL_F4(KERNEL, 32, f4, __VA_ARGS__) break;      \
    }

// hub rows (the a3 hub class, degree >= 1024) get kHubWarpsGat warps each; the rest a warp per row
constexpr int kHubWarpsGat = 8;

#define SS_HPL_F4B(KERNEL, H, f4, ...)                                                                        \
    switch (f4) {                                                                                             \
        case 1: launch_k(KERNEL<H, 1 __VA_ARGS__>, dim3(grid), dim3(256), 0, s, a); break;                    \
        case 2: launch_k(KERNEL<H, 2 __VA_ARGS__>, dim3(grid), dim3(256), 0, s, a); break;                    \
        case 3: launch_k(KERNEL<H, 3 __VA_ARGS__>, dim3(grid), dim3(256), 0, s, a); break;                    \
        case 4: launch_k(KERNEL<H, 4 __VA_ARGS__>, dim3(grid), dim3(256), 0, s, a); break;                    \
        case 5: launch_k(KERNEL<H, 5 __VA_ARGS__>, dim3(grid), dim3(256), 0, s, a); break;                    \
        case 6: launch_k(KERNEL<H, 6 __VA_ARGS__>, dim3(grid), dim3(256), 0, s, a); break;                    \
        case 7: launch_k(KERNEL<H, 7 __VA_ARGS__>, dim3(grid), dim3(256), 0, s, a); break;                    \
        default: launch_k(KERNEL<H, 8 __VA_ARGS__>, dim3(grid), dim3(256), 0, s, a); break;                   \
    }
#define SS_HPL_HB(KERNEL, H, f4, ...)                                \
    switch (H) {                                                     \
        case 2: SS_HPL_F4B(KERNEL, 2, f4, __VA_ARGS__) break;        \
        case 4: SS_HPL_F4B(KERNEL, 4, f4, __VA_ARGS__) break;        \
        case 8: SS_HPL_F4B(KERNEL, 8, f4, __VA_ARGS__) break;        \
        case 16: SS_HPL_F4B(KERNEL, 16, f4, __VA_ARGS__) break;      \
        default: SS_HPL_F4B(KERNEL, 32, f4, __VA_ARGS__) break;      \
    }

// the head-per-lane kernels read el at the compile-time row stride H (a runtime stride in the hot loop cost the
// layer-1 backward a spill reload and 50 % on Reddit, r2): an el packed into T's padding takes the generic kernels
bool launch_gat_fwd_hpl(const GatFwdArgs& a0, int64_t hub, cudaStream_t s) {
    const int f4 = hpl_f4(a0.H, a0.F, a0.ld, aligned16(a0.T) && aligned16(a0.A) && aligned16(a0.Y));
    if (!f4 || a0.ldel != a0.H) return false;
    static_assert(32 * kHubWarpsGat == 256, "long-row CTAs are the launch's 256-thread blocks");
    GatFwdArgs a = a0;
    a.nlong = std::min<int64_t>(std::max<int64_t>(hub - a0.row_begin, 0), a0.row_end - a0.row_begin);
    const unsigned grid = (unsigned)(a.nlong + (a.row_end - a.row_begin - a.nlong + 7) / 8);
    if (grid == 0) return true;
    if (a.nlong > 0) {                                 // long rows (a CTA each) + warp rows in one launch
        if (a.B) { SS_HPL_HB(k_gat_fwd_hpl, a.H, f4, , true, kHubWarpsGat) }
        else { SS_HPL_HB(k_gat_fwd_hpl, a.H, f4, , false, kHubWarpsGat) }
    } else {
        if (a.B) { SS_HPL_H(k_gat_fwd_hpl, a.H, f4, , true) }
        else { SS_HPL_H(k_gat_fwd_hpl, a.H, f4, , false) }
    }
    return true;
}

bool launch_gat_bwd_hpl(const GatBwdArgs& a0, int64_t hub, cudaStream_t s) {
    const int f4 = hpl_f4(a0.H, a0.F, a0.ldt, aligned16(a0.T) && aligned16(a0.D) && aligned16(a0.dT));
    if (!f4 || a0.ldel != a0.H) return false;
    GatBwdArgs a = a0;
    a.nlong = std::min<int64_t>(std::max<int64_t>(hub - a0.row_begin, 0), a0.row_end - a0.row_begin);
    const unsigned grid = (unsigned)(a.nlong + (a.row_end - a.row_begin - a.nlong + 7) / 8);
    if (grid == 0) return true;
    if (a.nlong > 0) { SS_HPL_HB(k_gat_bwd_hpl, a.H, f4, , kHubWarpsGat) }
    else { SS_HPL_H(k_gat_bwd_hpl, a.H, f4) }
    return true;
}

bool launch_gat_der_hpl(const GatBwdArgs& a, cudaStream_t s) {
    const int f4 = hpl_f4(a.H, a.F, a.ldt, aligned16(a.T) && aligned16(a.D));
    if (!f4 || a.ldel != a.H) return false;
    const unsigned grid = (unsigned)((a.row_end - a.row_begin + 7) / 8);
    if (grid) { SS_HPL_H(k_gat_der_hpl, a.H, f4) }
    return true;
}

}  // namespace seastar
