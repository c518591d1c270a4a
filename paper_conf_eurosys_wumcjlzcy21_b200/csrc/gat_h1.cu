// gat_h1.cu -- single-head GAT edge kernels (H = 1, any F <= 128, e.g. the output layer F = #classes):
// L lanes (<= 4) cover one edge and lane c owns the float4 chunks c, c + L, c + 2L, ... of the row
// (interleaved, so the L lanes' q-th loads are one contiguous 16L-byte span: each gathered row costs
// ~ceil(row bytes / 64) L1 wavefronts instead of one per lane-chunk), S = RL / L edge slots per row group; g = <dA, T> by an L-lane xor reduction.  PAPER.md Fig. 2 L95-L123,
// §6.3.4 L461-L463.  Same branch-free inner loop as gat_hpl.cu: an out-of-range edge slot gathers
// row 0 and gets weight 0; chunks past the row end are never loaded (per-lane constant predicate).
#include <algorithm>

#include "gat_common.cuh"

namespace seastar {

#ifndef GAT_H1_UBMAX
#define GAT_H1_UBMAX 4
#endif
template <int VPL>
#ifndef GAT_H1_UB3
#define GAT_H1_UB3 2        // edges per slot per batch at VPL = 3 (Reddit's F = 41 layer; A/B knob)
#endif
constexpr int h1_ub() {
    return (VPL <= 2 ? 4 : (VPL == 3 ? GAT_H1_UB3 : 2)) < GAT_H1_UBMAX ? (VPL <= 2 ? 4 : (VPL == 3 ? GAT_H1_UB3 : 2))
                                                                      : GAT_H1_UBMAX;
}

// load the lane's chunks of a row; chunks at or past W are zero (never loaded).  Columns inside
// the last partial chunk are loaded as stored (row padding): callers either zero the matching
// factor (own rows) or only read padding that is zero by construction (D records).
template <int VPL, int L>
__device__ __forceinline__ void load_lane_chunks(const float* p, const bool (&qv)[VPL], float4 (&x)[VPL]) {
#pragma unroll
    for (int q = 0; q < VPL; ++q) x[q] = qv[q] ? ldg4(p + 4 * L * q) : make_float4(0.f, 0.f, 0.f, 0.f);
}

// zero the columns >= nv of a chunk (nv in 0..4)
__device__ __forceinline__ float4 mask_tail(float4 x, int nv) {
    return make_float4(nv > 0 ? x.x : 0.f, nv > 1 ? x.y : 0.f, nv > 2 ? x.z : 0.f, nv > 3 ? x.w : 0.f);
}

// WPR > 1 (RL = 32): the launch's first a.nlong blocks each own one long row, warp w over the w-th contiguous slice
// of the row's edges, slices merged in warp order by the online-softmax merge through shared memory; later blocks
// own 8 warp rows (as k_gat_fwd_hpl)
template <int VPL, int L, int RL, bool SB, int WPR = 1>
#ifndef GAT_MB_FWD_H1
#define GAT_MB_FWD_H1 GAT_MB_FWD
#endif
__global__ void __launch_bounds__(256, GAT_MB_FWD_H1) k_gat_fwd_h1(const GatFwdArgs a) {
    static_assert(WPR == 1 || RL == 32, "hub rows take whole warps");
    constexpr int NV = 4 * VPL, S = RL / L;
    constexpr int UE = h1_ub<VPL>() < L ? h1_ub<VPL>() : L;   // edges per slot per batch
    constexpr int NB = L / UE;                                 // batches per RL-edge chunk
    constexpr int NP = SB ? NV : 1;
    const int lane = threadIdx.x & 31;
    const int gl = lane % RL, slot = gl / L, c = gl % L;
    const unsigned gmask = (RL == 32) ? 0xffffffffu : (((1u << RL) - 1u) << ((lane / RL) * RL));
    const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int wib = threadIdx.x >> 5;
    const bool hubblk = WPR > 1 && (int64_t)blockIdx.x < a.nlong;      // block-uniform
    const int64_t row = hubblk ? a.row_begin + blockIdx.x
                      : WPR > 1 ? a.row_begin + a.nlong + ((int64_t)blockIdx.x - a.nlong) * (blockDim.x >> 5) + wib
                                : a.row_begin + warp * (32 / RL) + lane / RL;
    const bool valid = row < a.row_end;
    int beg = valid ? __ldg(a.off + row) : 0;
    int end = valid ? __ldg(a.off + row + 1) : 0;
    if (hubblk) {
        const int64_t len = end - beg;
        const int b0 = beg + (int)(len * wib / WPR);
        end = beg + (int)(len * (wib + 1) / WPR);
        beg = b0;
    }
    const int64_t v = valid ? (int64_t)__ldg(a.perm + row) - a.vbase : 0;
    const int W = a.F, col0 = 4 * c;             // chunk q of this lane: columns col0 + 4 L q ..
    bool qv[VPL];
#pragma unroll
    for (int q = 0; q < VPL; ++q) qv[q] = col0 + 4 * L * q < W;
    const float erv = valid ? __ldg(a.er + v) : 0.f;
    const float slope = a.slope;
    const float* Tc = a.T + col0;
    float m = kNegBig, mlog = kNegBig * kLog2e, ssum = 0.f, psum = 0.f;
    float acc[NV], pacc[NP];
#pragma unroll
    for (int i = 0; i < NV; ++i) acc[i] = 0.f;
#pragma unroll
    for (int i = 0; i < NP; ++i) pacc[i] = 0.f;
    int nxt = (gl < end - beg) ? __ldcs(a.nbr + beg + gl) : 0;
    for (int base = beg; base < end; base += RL) {
        const int n = min(RL, end - base);
        const int my = nxt;
        nxt = (gl < end - base - RL) ? __ldcs(a.nbr + base + RL + gl) : 0;
#pragma unroll
        for (int b = 0; b < NB; ++b) {
            if (b * UE * S >= n) break;
            float z[UE];
            float4 x[UE][VPL];
#pragma unroll
            for (int jj = 0; jj < UE; ++jj) {
                const int k = (b * UE + jj) * S + slot;     // < RL
                const int u = __shfl_sync(gmask, my, k, RL);
                load_lane_chunks<VPL, L>(row_ptr(Tc, u, a.ld), qv, x[jj]);
                const float s = __ldg(a.el + (size_t)(uint32_t)u * (size_t)a.ldel) + erv;
                z[jj] = k < n ? lrelu(s, slope) : -INFINITY;
            }
            float mb = m;
#pragma unroll
            for (int jj = 0; jj < UE; ++jj) mb = fmaxf(mb, z[jj]);
            if (mb > m) {
                const float corr = ex2((m - mb) * kLog2e);
                ssum *= corr;
#pragma unroll
                for (int i = 0; i < NV; ++i) acc[i] *= corr;
                if (SB) {
                    psum *= corr;
#pragma unroll
                    for (int i = 0; i < NP; ++i) pacc[i] *= corr;
                }
                m = mb;
                mlog = mb * kLog2e;
            }
#pragma unroll
            for (int jj = 0; jj < UE; ++jj) {
                const float p = ex2(fmaf(z[jj], kLog2e, -mlog));
                ssum += p;
#pragma unroll
                for (int q = 0; q < VPL; ++q) {
                    acc[4 * q] = fmaf(p, x[jj][q].x, acc[4 * q]);
                    acc[4 * q + 1] = fmaf(p, x[jj][q].y, acc[4 * q + 1]);
                    acc[4 * q + 2] = fmaf(p, x[jj][q].z, acc[4 * q + 2]);
                    acc[4 * q + 3] = fmaf(p, x[jj][q].w, acc[4 * q + 3]);
                }
                if (SB) {
                    const float pp = z[jj] > 0.f ? p : 0.f;
                    psum += pp;
#pragma unroll
                    for (int q = 0; q < (SB ? VPL : 0); ++q) {
                        pacc[(4 * q) % NP] = fmaf(pp, x[jj][q].x, pacc[(4 * q) % NP]);
                        pacc[(4 * q + 1) % NP] = fmaf(pp, x[jj][q].y, pacc[(4 * q + 1) % NP]);
                        pacc[(4 * q + 2) % NP] = fmaf(pp, x[jj][q].z, pacc[(4 * q + 2) % NP]);
                        pacc[(4 * q + 3) % NP] = fmaf(pp, x[jj][q].w, pacc[(4 * q + 3) % NP]);
                    }
                }
            }
        }
    }
#pragma unroll
    for (int o = L; o < RL; o <<= 1) {
        const float mo = __shfl_xor_sync(gmask, m, o, RL);
        const float so = __shfl_xor_sync(gmask, ssum, o, RL);
        const float mn = fmaxf(m, mo);
        const float ca = ex2((m - mn) * kLog2e), cb = ex2((mo - mn) * kLog2e);
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
    if (hubblk) {                                       // merge the warps' slices in warp order
        constexpr int NS = 3 + NV + (SB ? NP : 0);
        __shared__ float st[WPR > 1 ? WPR : 1][L][NS];
        if (slot == 0) {
            float* p = st[wib][c];
            p[0] = m; p[1] = ssum; p[2] = psum;
#pragma unroll
            for (int i = 0; i < NV; ++i) p[3 + i] = acc[i];
#pragma unroll
            for (int i = 0; i < (SB ? NP : 0); ++i) p[3 + NV + i] = pacc[i];
        }
        __syncthreads();
        if (wib != 0) return;
        if (slot == 0)
            for (int w2 = 1; w2 < WPR; ++w2) {
                const float* p = st[w2][c];
                const float mo = p[0], mn = fmaxf(m, mo);
                const float ca = ex2((m - mn) * kLog2e), cb = ex2((mo - mn) * kLog2e);
                ssum = ssum * ca + p[1] * cb;
#pragma unroll
                for (int i = 0; i < NV; ++i) acc[i] = acc[i] * ca + p[3 + i] * cb;
                if (SB) {
                    psum = psum * ca + p[2] * cb;
#pragma unroll
                    for (int i = 0; i < NP; ++i) pacc[i] = pacc[i] * ca + p[3 + NV + (SB ? i : 0)] * cb;
                }
                m = mn;
            }
    }
    if (!valid || slot != 0) return;
    const float inv = ssum > 0.f ? 1.f / ssum : 0.f;
    float* pa = a.A + v * a.ld;
    float* py = a.Y + v * a.ld;
    float* pb = SB ? a.B + v * a.ld : nullptr;
#pragma unroll
    for (int q = 0; q < VPL; ++q) {
        const int col = col0 + 4 * L * q;
        if (col >= W) continue;
        float o4[4], y4[4], b4[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            o4[i] = acc[4 * q + i] * inv;
            y4[i] = act_apply(a.act, o4[i] + ((a.bias && col + i < W) ? __ldg(a.bias + col + i) : 0.f));
            b4[i] = SB ? slope * o4[i] + (1.f - slope) * pacc[(4 * q + i) % NP] * inv : 0.f;
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
        if (SB) a.bsum[v] = ssum > 0.f ? slope + (1.f - slope) * psum * inv : 0.f;
    }
}

// DER = false: source-major dT/del over REV (own = T_u, gathered = records D[v]);
// DER = true: destination-major der over FWD (own = dA_v from D[v], gathered = T_u)
#ifndef GAT_MB_BWD_H1
#define GAT_MB_BWD_H1 GAT_MB_BWD
#endif
#ifndef GAT_H1_BWD_UBMAX
#define GAT_H1_BWD_UBMAX 4
#endif
// VPL = 3 (Reddit's F = 41 layer): 4 edges per slot per batch at 2 blocks per SM (124 registers) -- measured
// (tools/ab_reddit.sh): layer-2 backward 1.905 -> 1.833 ms; the forward keeps 2 edges at 3 blocks (4 edges: 2.00 ->
// 2.44 ms at 2 blocks, spills at 3)
#ifndef GAT_H1_BWD_UB3
#define GAT_H1_BWD_UB3 4
#endif
#ifndef GAT_MB_BWD_H1_V3
#define GAT_MB_BWD_H1_V3 2
#endif
template <int VPL, int L, int RL, bool DER, int WPR = 1>
__global__ void __launch_bounds__(256, VPL == 3 ? GAT_MB_BWD_H1_V3 : GAT_MB_BWD_H1) k_gat_bwd_h1(const GatBwdArgs a) {
    static_assert(WPR == 1 || RL == 32, "hub rows take whole warps");
    constexpr int NV = 4 * VPL, S = RL / L;
    constexpr int UBV = VPL == 3 ? GAT_H1_BWD_UB3 : h1_ub<VPL>();
    constexpr int UB0 = UBV < GAT_H1_BWD_UBMAX ? UBV : GAT_H1_BWD_UBMAX;
    constexpr int UE = UB0 < L ? UB0 : L;
    constexpr int NB = L / UE;
    const int lane = threadIdx.x & 31;
    const int gl = lane % RL, slot = gl / L, c = gl % L;
    const unsigned gmask = (RL == 32) ? 0xffffffffu : (((1u << RL) - 1u) << ((lane / RL) * RL));
    const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int wib = threadIdx.x >> 5;
    const bool hubblk = WPR > 1 && (int64_t)blockIdx.x < a.nlong;      // block-uniform
    const int64_t row = hubblk ? a.row_begin + blockIdx.x
                      : WPR > 1 ? a.row_begin + a.nlong + ((int64_t)blockIdx.x - a.nlong) * (blockDim.x >> 5) + wib
                                : a.row_begin + warp * (32 / RL) + lane / RL;
    const bool valid = row < a.row_end;
    int beg = valid ? __ldg(a.off + row) : 0;
    int end = valid ? __ldg(a.off + row + 1) : 0;
    if (hubblk) {                                       // long rows: warp w takes the w-th slice
        const int64_t len = end - beg;
        const int b0 = beg + (int)(len * wib / WPR);
        end = beg + (int)(len * (wib + 1) / WPR);
        beg = b0;
    }
    const int64_t w = valid ? (int64_t)__ldg(a.perm + row) - a.vbase : 0;   // u (src-major) or v (der)
    const int W = a.F, col0 = 4 * c;             // chunk q of this lane: columns col0 + 4 L q ..
    const int aux0 = rec_aux_offset(W);
    const float slope = a.slope;
    bool qv[VPL];
#pragma unroll
    for (int q = 0; q < VPL; ++q) qv[q] = valid && col0 + 4 * L * q < W;
    // own row, padding columns zeroed so gathered padding never enters g
    float4 own[VPL];
    float4 k4 = make_float4(0.f, 0.f, 0.f, 0.f);   // src-major: (el_u, -, -, -); der: (er, lse, c, nl2)_v
    if (!DER) {
        load_lane_chunks<VPL, L>(a.T + w * a.ldt + col0, qv, own);
        if (valid) k4.x = __ldg(a.el + w * a.ldel);
    } else {
        load_lane_chunks<VPL, L>(a.D + w * a.ldd + col0, qv, own);
        if (valid) k4 = ldg4(a.D + w * a.ldd + aux0);
    }
    int nvalid[VPL];   // valid columns of each chunk (0..4)
#pragma unroll
    for (int q = 0; q < VPL; ++q) {
        nvalid[q] = min(4, max(0, W - (col0 + 4 * L * q)));
        own[q] = mask_tail(own[q], nvalid[q]);
    }
    const float* Gc = DER ? a.T + col0 : a.D + col0;           // gathered rows
    const int64_t gld = DER ? a.ldt : a.ldd;
    float acc[NV], dsum = 0.f;
#pragma unroll
    for (int i = 0; i < NV; ++i) acc[i] = 0.f;
    int nxt = (gl < end - beg) ? __ldcs(a.nbr + beg + gl) : 0;
    for (int base = beg; base < end; base += RL) {
        const int n = min(RL, end - base);
        const int my = nxt;
        nxt = (gl < end - base - RL) ? __ldcs(a.nbr + base + RL + gl) : 0;
#pragma unroll
        for (int b = 0; b < NB; ++b) {
            if (b * UE * S >= n) break;
            float4 x[UE][VPL];
            float4 e[UE];
            int kk[UE];
#pragma unroll
            for (int jj = 0; jj < UE; ++jj) {
                kk[jj] = (b * UE + jj) * S + slot;
                const int o = __shfl_sync(gmask, my, kk[jj], RL);
                load_lane_chunks<VPL, L>(row_ptr(Gc, o, gld), qv, x[jj]);
                if (!DER) {
                    e[jj] = ldg4(row_ptr(a.D + aux0, o, a.ldd));          // (er, lse, c, nl2)_v
                } else {
                    e[jj] = make_float4(__ldg(a.el + (size_t)(uint32_t)o * (size_t)a.ldel), 0.f, 0.f, 0.f);  // el_u
                    // gathered T rows may carry non-finite padding (NaN * 0 = NaN): zero it
#pragma unroll
                    for (int q = 0; q < VPL; ++q) x[jj][q] = mask_tail(x[jj][q], nvalid[q]);
                }
            }
#pragma unroll
            for (int jj = 0; jj < UE; ++jj) {
                float g = 0.f;
#pragma unroll
                for (int q = 0; q < VPL; ++q) {
                    g = fmaf(x[jj][q].x, own[q].x, g);
                    g = fmaf(x[jj][q].y, own[q].y, g);
                    g = fmaf(x[jj][q].z, own[q].z, g);
                    g = fmaf(x[jj][q].w, own[q].w, g);
                }
#pragma unroll
                for (int o = 1; o < L; o <<= 1) g += __shfl_xor_sync(gmask, g, o, RL);
                // s = el_u + er_v ; alpha = exp(LReLU(s) - lse_v) ; ds = alpha (g - c_v) LReLU'(s)
                const float s = DER ? e[jj].x + k4.x : k4.x + e[jj].x;
                const float nl2 = DER ? k4.w : e[jj].w;
                const float cv = DER ? k4.z : e[jj].z;
                const bool pos = s > 0.f;
                const float al0 = ex2(fmaf(pos ? s : slope * s, kLog2e, nl2));
                const float al = kk[jj] < n ? al0 : 0.f;
                dsum = fmaf(al * (g - cv), pos ? 1.f : slope, dsum);
                if (!DER) {
#pragma unroll
                    for (int q = 0; q < VPL; ++q) {
                        acc[4 * q] = fmaf(al, x[jj][q].x, acc[4 * q]);
                        acc[4 * q + 1] = fmaf(al, x[jj][q].y, acc[4 * q + 1]);
                        acc[4 * q + 2] = fmaf(al, x[jj][q].z, acc[4 * q + 2]);
                        acc[4 * q + 3] = fmaf(al, x[jj][q].w, acc[4 * q + 3]);
                    }
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
    if (hubblk) {                                       // add the warps' slices in warp order
        __shared__ float st[WPR > 1 ? WPR : 1][L][NV + 1];
        if (slot == 0) {
#pragma unroll
            for (int i = 0; i < NV; ++i) st[wib][c][i] = DER ? 0.f : acc[i];
            st[wib][c][NV] = dsum;
        }
        __syncthreads();
        if (wib != 0) return;
        if (slot == 0)
            for (int w2 = 1; w2 < WPR; ++w2) {
                if (!DER)
#pragma unroll
                    for (int i = 0; i < NV; ++i) acc[i] += st[w2][c][i];
                dsum += st[w2][c][NV];
            }
    }
    if (!valid || slot != 0) return;
    if (DER) {
        if (c == 0) a.der[w] = dsum;
        return;
    }
    float* pd = a.dT + w * a.ldt;
#pragma unroll
    for (int q = 0; q < VPL; ++q) {
        const int col = col0 + 4 * L * q;
        if (col >= W) continue;
        if (col + 4 <= W)
            *reinterpret_cast<float4*>(pd + col) = make_float4(acc[4 * q], acc[4 * q + 1], acc[4 * q + 2], acc[4 * q + 3]);
        else
            for (int i = 0; i < 4 && col + i < W; ++i) pd[col + i] = acc[4 * q + i];
    }
    if (c == 0) a.del[w] = dsum;
}

// ---------------------------------------------------------------------------------------------
// launchers over the two degree classes: warp rows (RL = 32, degree >= 32) and 4-lane row groups
// ---------------------------------------------------------------------------------------------
constexpr int kHubWarpsH1 = 8;      // warps per hub row (degree >= 1024)

// degree classes: [0, split) warp rows (degree >= 32; the first `hub` of them long rows with a CTA each),
// [split, mid) 16-lane row groups (8 <= degree < 32: 16 / L edges in flight per row instead of one slot of 4 lanes --
// the small graphs' latency-bound class, r2), [mid, n_rows) 4-lane row groups
template <typename Args, typename LH, typename LW, typename LM, typename LS>
static void h1_buckets(const Args& a, int64_t hub, int64_t split, int64_t mid, int64_t n_rows, LH lh, LW lw, LM lm,
                       LS ls) {
    Args hi = a, md = a, lo = a;
    mid = std::min<int64_t>(std::max<int64_t>(mid, split), n_rows);
    hi.row_begin = 0; hi.row_end = split;
    hi.nlong = std::min<int64_t>(hub, split);
    md.row_begin = split; md.row_end = mid; md.nlong = 0;
    lo.row_begin = mid; lo.row_end = n_rows;
    lo.nlong = 0;
    if (split > 0) {
        const unsigned g = (unsigned)(hi.nlong + (split - hi.nlong + 7) / 8);
        if (hi.nlong > 0) lh(hi, g);                                        // long rows + warp rows, one launch
        else lw(hi, g);
    }
    if (mid > split) lm(md, (unsigned)((mid - split + 15) / 16));          // RL = 16: 16 rows per block
    if (n_rows > mid) ls(lo, (unsigned)((n_rows - mid + 63) / 64));       // RL = 4: 64 rows per block
}

template <int VPL, int L>
static void fwd_h1_run(const GatFwdArgs& a, int64_t hub, int64_t split, int64_t mid, int64_t n, cudaStream_t s) {
    if (a.B)
        h1_buckets(a, hub, split, mid, n,
                   [&](const GatFwdArgs& x, unsigned g) { launch_k(k_gat_fwd_h1<VPL, L, 32, true, kHubWarpsH1>, dim3(g), dim3(32 * kHubWarpsH1), 0, s, x); },
                   [&](const GatFwdArgs& x, unsigned g) { launch_k(k_gat_fwd_h1<VPL, L, 32, true>, dim3(g), dim3(256), 0, s, x); },
                   [&](const GatFwdArgs& x, unsigned g) { launch_k(k_gat_fwd_h1<VPL, L, 16, true>, dim3(g), dim3(256), 0, s, x); },
                   [&](const GatFwdArgs& x, unsigned g) { launch_k(k_gat_fwd_h1<VPL, L, 4, true>, dim3(g), dim3(256), 0, s, x); });
    else
        h1_buckets(a, hub, split, mid, n,
                   [&](const GatFwdArgs& x, unsigned g) { launch_k(k_gat_fwd_h1<VPL, L, 32, false, kHubWarpsH1>, dim3(g), dim3(32 * kHubWarpsH1), 0, s, x); },
                   [&](const GatFwdArgs& x, unsigned g) { launch_k(k_gat_fwd_h1<VPL, L, 32, false>, dim3(g), dim3(256), 0, s, x); },
                   [&](const GatFwdArgs& x, unsigned g) { launch_k(k_gat_fwd_h1<VPL, L, 16, false>, dim3(g), dim3(256), 0, s, x); },
                   [&](const GatFwdArgs& x, unsigned g) { launch_k(k_gat_fwd_h1<VPL, L, 4, false>, dim3(g), dim3(256), 0, s, x); });
}

template <int VPL, int L>
static void bwd_h1_run(const GatBwdArgs& a, int64_t hub, int64_t split, int64_t mid, int64_t n, bool der,
                       cudaStream_t s) {
    if (der)
        h1_buckets(a, hub, split, mid, n,
                   [&](const GatBwdArgs& x, unsigned g) { launch_k(k_gat_bwd_h1<VPL, L, 32, true, kHubWarpsH1>, dim3(g), dim3(32 * kHubWarpsH1), 0, s, x); },
                   [&](const GatBwdArgs& x, unsigned g) { launch_k(k_gat_bwd_h1<VPL, L, 32, true>, dim3(g), dim3(256), 0, s, x); },
                   [&](const GatBwdArgs& x, unsigned g) { launch_k(k_gat_bwd_h1<VPL, L, 16, true>, dim3(g), dim3(256), 0, s, x); },
                   [&](const GatBwdArgs& x, unsigned g) { launch_k(k_gat_bwd_h1<VPL, L, 4, true>, dim3(g), dim3(256), 0, s, x); });
    else
        h1_buckets(a, hub, split, mid, n,
                   [&](const GatBwdArgs& x, unsigned g) { launch_k(k_gat_bwd_h1<VPL, L, 32, false, kHubWarpsH1>, dim3(g), dim3(32 * kHubWarpsH1), 0, s, x); },
                   [&](const GatBwdArgs& x, unsigned g) { launch_k(k_gat_bwd_h1<VPL, L, 32, false>, dim3(g), dim3(256), 0, s, x); },
                   [&](const GatBwdArgs& x, unsigned g) { launch_k(k_gat_bwd_h1<VPL, L, 16, false>, dim3(g), dim3(256), 0, s, x); },
                   [&](const GatBwdArgs& x, unsigned g) { launch_k(k_gat_bwd_h1<VPL, L, 4, false>, dim3(g), dim3(256), 0, s, x); });
}

#define SS_H1_DISPATCH(RUN, vpl, L, ...)                                          \
    switch (vpl * 8 + L) {                                                        \
        case 1 * 8 + 1: RUN<1, 1>(__VA_ARGS__); break;                            \
        case 1 * 8 + 2: RUN<1, 2>(__VA_ARGS__); break;                            \
        case 1 * 8 + 4: RUN<1, 4>(__VA_ARGS__); break;                            \
        case 2 * 8 + 1: RUN<2, 1>(__VA_ARGS__); break;                            \
        case 2 * 8 + 2: RUN<2, 2>(__VA_ARGS__); break;                            \
        case 2 * 8 + 4: RUN<2, 4>(__VA_ARGS__); break;                            \
        case 3 * 8 + 1: RUN<3, 1>(__VA_ARGS__); break;                            \
        case 3 * 8 + 2: RUN<3, 2>(__VA_ARGS__); break;                            \
        case 3 * 8 + 4: RUN<3, 4>(__VA_ARGS__); break;                            \
        case 4 * 8 + 1: RUN<4, 1>(__VA_ARGS__); break;                            \
        case 4 * 8 + 2: RUN<4, 2>(__VA_ARGS__); break;                            \
        case 4 * 8 + 4: RUN<4, 4>(__VA_ARGS__); break;                            \
        case 6 * 8 + 1: RUN<6, 1>(__VA_ARGS__); break;                            \
        case 6 * 8 + 2: RUN<6, 2>(__VA_ARGS__); break;                            \
        case 6 * 8 + 4: RUN<6, 4>(__VA_ARGS__); break;                            \
        case 8 * 8 + 1: RUN<8, 1>(__VA_ARGS__); break;                            \
        case 8 * 8 + 2: RUN<8, 2>(__VA_ARGS__); break;                            \
        default: RUN<8, 4>(__VA_ARGS__); break;                                   \
    }

bool launch_gat_fwd_h1(const GatFwdArgs& a, int64_t hub, int64_t split, int64_t mid, int64_t n_rows, cudaStream_t s) {
    int vpl = 0, L = 0;
    if (!h1_geometry(a.H, a.F, a.ld, aligned16(a.T) && aligned16(a.A) && aligned16(a.Y), vpl, L)) return false;
    SS_H1_DISPATCH(fwd_h1_run, vpl, L, a, hub, split, mid, n_rows, s)
    return true;
}

bool launch_gat_bwd_h1(const GatBwdArgs& a, int64_t hub, int64_t split, int64_t mid, int64_t n_rows, bool der,
                       cudaStream_t s) {
    int vpl = 0, L = 0;
    const bool al = der ? aligned16(a.T) && aligned16(a.D) : aligned16(a.T) && aligned16(a.D) && aligned16(a.dT);
    if (!h1_geometry(a.H, a.F, a.ldt, al, vpl, L)) return false;
    SS_H1_DISPATCH(bwd_h1_run, vpl, L, a, hub, split, mid, n_rows, der, s)
    return true;
}

}  // namespace seastar
