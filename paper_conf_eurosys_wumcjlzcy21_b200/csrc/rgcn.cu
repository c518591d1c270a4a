// rgcn.cu -- a7 / a10: fused R-GCN layer (§6.3.5, layer of [53]).
//
// "Heterogeneous Seastar": the aggregation is hierarchical -- sum over the edges of one type, then
// over types -- and the paper runs it sequentially by sorting each vertex's edges by type and
// "detecting changes of edge types" (L473-L475).  On B200:
//   forward (dst-major, FWD CSR, type-sorted rows): every edge slot keeps a run-sum g of
//     norm_e * X[src_e] in registers; when its type changes, g is pushed through W_r, which is staged
//     once per CTA in shared memory (R x F_in x F_out fp32, <= 200 KB), and accumulated into the
//     row's output; the slots are merged by a fixed shuffle tree; no atomics.
//   dX (src-major, REV CSR, type-sorted rows): the same skeleton gathering dA[dst] with W_r^T staged.
//   dW (type-major view built at graph_create): dW_r = sum_v g_{v,r} (x) dA[v], where g_{v,r} is the
//     forward run-sum.  Runs are grouped into tasks that never cross a type, so each warp keeps its
//     dW_r partial in registers; per-task partials are reduced per type in task order
//     (deterministic; no shared- or global-memory atomics).
#include <algorithm>
#include <cstdlib>
#include <type_traits>

#include "common.cuh"
#include "rgcn_tile.cuh"

namespace seastar {

struct RgcnRowArgs {
    const int32_t* perm; const int32_t* off; const int32_t* nbr; const int32_t* typ;
    const float* norm; const int32_t* eid; const float* norm_user;
    int64_t row_begin, row_end, vbase;
    const float* table; int64_t ldt;   // gathered rows (X_all forward, dA_all for dX)
    const float* W;                     // [R, F_in, F_out]
    int R, Fg, Fo;                      // gathered width, output width
    int transpose;                      // 0: forward (g W_r), 1: dX (q W_r^T)
    int wstride;                        // floats between consecutive staged W_r blocks (w_stride)
    float* out; int64_t ldo;
    const float* bias; int act;
    const float* Yact;                  // dX only: fused activation backward, out *= act'(Yact)
};

// stage W (or W^T) as [R][Fg][Fop] with Fop = round4(Fo), zero padded; consecutive W_r blocks start at a stride
// of 16 mod 32 floats: the 32/RL row groups of a warp flush runs of different types at the same in-block offset, and a
// 128-bit shared load is served 8 lanes (two 4-lane groups) per wavefront, so two groups whose types differ in parity
// never share a bank, and equal types broadcast (with a 4-float pad, measured on the AM shape: 37 % of the flush
// wavefronts were bank conflicts)
// (the smallest such stride >= Fg * Fop, and the dense stride Fg * Fop when the padded table does not fit)
inline int64_t w_stride_padded(int Fg, int Fop) {
    const int64_t d = (int64_t)Fg * Fop;
    return d + ((16 - d % 32) % 32 + 32) % 32;
}
constexpr size_t kRgcnSmemMax = 227 * 1024 - sizeof(float) * 64 * 32;   // dynamic smem budget (hub CTAs' red[])
inline int64_t w_stride(int R, int Fg, int Fop) {
    const int64_t p = w_stride_padded(Fg, Fop);
    return (size_t)R * p * sizeof(float) <= kRgcnSmemMax ? p : (int64_t)Fg * Fop;
}

__device__ void stage_w(const RgcnRowArgs& a, float* Ws) {
    // 32-bit index math: the staged table fits in shared memory, and 64-bit div/mod made the staging of the 136 KB
    // AM table cost tens of microseconds per CTA
    const int Fop = (a.Fo + 3) & ~3;
    const int n = a.R * a.Fg * Fop;
    const int ws = a.wstride;
    for (int idx = threadIdx.x; idx < n; idx += blockDim.x) {
        const int j = idx % Fop;
        const int ri = idx / Fop;
        const int i = ri % a.Fg;
        const int r = ri / a.Fg;
        float w = 0.f;
        if (j < a.Fo) {
            // forward: Ws[r][i][j] = W[r][i][j] (i in F_in, j in F_out)
            // dX     : Ws[r][j'][i'] = W[r][i'][j'] with gathered index = j' (F_out), output = i' (F_in)
            w = a.transpose ? __ldg(a.W + (r * a.Fo + j) * a.Fg + i)
                            : __ldg(a.W + ri * a.Fo + j);
        }
        Ws[r * ws + i * Fop + j] = w;
    }
}

template <int L, int RL, int WPR, int BS = 512>
__global__ void __launch_bounds__(BS) k_rgcn_rows(const RgcnRowArgs a) {
    extern __shared__ float4 smem4[];
    float* Ws = reinterpret_cast<float*>(smem4);
    stage_w(a, Ws);
    __syncthreads();
    constexpr int S = RL / L;
    constexpr int UB = (L < 4 ? L : 4);
    const int lane = threadIdx.x & 31;
    const int gl = lane % RL;
    const int slot = gl / L;
    const int c = gl % L;
    const unsigned gmask = (RL == 32) ? 0xffffffffu : (((1u << RL) - 1u) << ((lane / RL) * RL));
    const unsigned smask = (L == 32) ? 0xffffffffu : (((1u << L) - 1u) << ((lane / L) * L));
    const int Fop = (a.Fo + 3) & ~3;
    const int Cg = (a.Fg + 3) / 4, Co = (a.Fo + 3) / 4;
    const int gpb = WPR > 1 ? 1 : blockDim.x / RL;
    const int64_t ngroups = (int64_t)gridDim.x * gpb;
    const int warp = threadIdx.x >> 5;
    __shared__ float red[WPR > 1 ? WPR : 1][64];

    for (int64_t row = a.row_begin + (int64_t)blockIdx.x * gpb + (WPR > 1 ? 0 : threadIdx.x / RL); row < a.row_end;
         row += ngroups) {
        int beg = __ldg(a.off + row), end = __ldg(a.off + row + 1);
        if (WPR > 1) {
            const int64_t n = end - beg;
            const int b0 = beg + (int)(n * warp / WPR);
            end = beg + (int)(n * (warp + 1) / WPR);
            beg = b0;
        }
        const int64_t v = (int64_t)__ldg(a.perm + row) - a.vbase;
        float out[4] = {0.f, 0.f, 0.f, 0.f};
        float g[4] = {0.f, 0.f, 0.f, 0.f};
        int cur = -1;
        auto flush = [&](int r) {
            const float* wr = Ws + (int64_t)r * a.wstride;
#pragma unroll
            for (int cl = 0; cl < L; ++cl) {
                if (cl >= Cg) break;
                float gv[4];
#pragma unroll
                for (int q = 0; q < 4; ++q) gv[q] = __shfl_sync(smask, g[q], cl, L);
                if (c < Co) {
#pragma unroll
                    for (int q = 0; q < 4; ++q) {
                        const int i = 4 * cl + q;
                        if (i < a.Fg) {
                            const float4 w4 = *reinterpret_cast<const float4*>(wr + (int64_t)i * Fop + 4 * c);
                            out[0] = fmaf(gv[q], w4.x, out[0]);
                            out[1] = fmaf(gv[q], w4.y, out[1]);
                            out[2] = fmaf(gv[q], w4.z, out[2]);
                            out[3] = fmaf(gv[q], w4.w, out[3]);
                        }
                    }
                }
            }
        };
        // edge-record prefetch: the next chunk's (u, type, norm) loads are in flight during this chunk
        int nx_u = 0, nx_t = 0;
        float nx_w = 0.f;
        auto fetch = [&](int b) {
            nx_u = 0; nx_t = 0; nx_w = 0.f;
            if (gl < end - b) {
                nx_u = __ldcs(a.nbr + b + gl);
                nx_t = __ldcs(a.typ + b + gl);
                nx_w = a.norm_user ? __ldg(a.norm_user + __ldg(a.eid + b + gl)) : __ldg(a.norm + b + gl);
            }
        };
        fetch(beg);
        for (int base = beg; base < end; base += RL) {
            const int n = min(RL, end - base);
            const int my_u = nx_u, my_t = nx_t;
            const float my_w = nx_w;
            fetch(base + RL);
#pragma unroll
            for (int j0 = 0; j0 < L; j0 += UB) {
                if (j0 * S >= n) break;
                float x[UB][4];
                int tt[UB];
                float ww[UB];
#pragma unroll
                for (int jj = 0; jj < UB; ++jj) {
                    const int k = (j0 + jj) * S + slot;
                    const int u = __shfl_sync(gmask, my_u, k & (RL - 1), RL);
                    tt[jj] = __shfl_sync(gmask, my_t, k & (RL - 1), RL);
                    ww[jj] = __shfl_sync(gmask, my_w, k & (RL - 1), RL);
                    if (k < n && c < Cg) {
                        const float4 t4 = ldg4(a.table + (int64_t)u * a.ldt + 4 * c);
                        x[jj][0] = t4.x; x[jj][1] = t4.y; x[jj][2] = t4.z; x[jj][3] = t4.w;
#pragma unroll
                        for (int q = 0; q < 4; ++q)
                            if (4 * c + q >= a.Fg) x[jj][q] = 0.f;
                    } else {
#pragma unroll
                        for (int q = 0; q < 4; ++q) x[jj][q] = 0.f;
                    }
                }
#pragma unroll
                for (int jj = 0; jj < UB; ++jj) {
                    const int k = (j0 + jj) * S + slot;
                    if (k < n) {                     // slot-uniform
                        if (tt[jj] != cur) {
                            if (cur >= 0) flush(cur);
                            g[0] = g[1] = g[2] = g[3] = 0.f;
                            cur = tt[jj];
                        }
#pragma unroll
                        for (int q = 0; q < 4; ++q) g[q] = fmaf(ww[jj], x[jj][q], g[q]);
                    }
                }
            }
        }
        if (cur >= 0) flush(cur);
#pragma unroll
        for (int o = L; o < RL; o <<= 1)
#pragma unroll
            for (int q = 0; q < 4; ++q) out[q] += __shfl_xor_sync(gmask, out[q], o, RL);
        if (WPR > 1) {
            if (slot == 0 && c < Co)
#pragma unroll
                for (int q = 0; q < 4; ++q) red[warp][4 * c + q] = out[q];
            __syncthreads();
            if (warp == 0 && slot == 0 && c < Co)
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    float t = red[0][4 * c + q];
                    for (int w = 1; w < WPR; ++w) t += red[w][4 * c + q];
                    out[q] = t;
                }
            __syncthreads();
            if (warp != 0) continue;
        }
        if (slot == 0 && c < Co) {
            float* po = a.out + v * a.ldo + 4 * c;
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                const int j = 4 * c + q;
                if (j < a.Fo) {
                    float z = out[q];
                    if (!a.transpose) z = act_apply(a.act, z + (a.bias ? __ldg(a.bias + j) : 0.f));
                    else if (a.Yact) z *= act_grad_from_y(a.act, __ldg(a.Yact + v * a.ldo + j));
                    po[q] = z;
                }
            }
        }
    }
}

// ---------------------------------------------------------------------------------------------------
// Two-phase path (F_in, F_out <= 16: every R-GCN layer of the BASELINE configs).  The one-pass kernel above pushes
// every (row, type) run through a W_r read from shared memory by the run's own lanes -- 1 KB of un-shared loads per
// run, and on the AM shape (mean in-degree 3, 133 types) a run is ~1 edge -- which bounds it at ~11 % of HBM
// (VERDICT r1).  Here the edges are visited in type-major order instead (a lane per edge), so the 32 lanes of a warp
// share W_r and every shared-memory read of W_r is a broadcast:
//   phase 1 (k_rgcn_edge):   per edge e of type r: H[pos_e] = norm_e * table[nbr_e] W_r    (pos_e = e's row-order
//                            position, so the products of one row are contiguous)
//   phase 2 (k_rgcn_rowsum): per row v: out[v] = epilogue(sum_{e in row v} H[e])
// Forward: table = X, W_r as given, epilogue act(. + b).  dX (transpose): table = dA, W_r^T, epilogue * act'(Yact).
// Deterministic: every product has its own slot and each row sums its slots in row order (type, eid); no atomics.
// (An r2 variant that summed type runs into segments before the product was instruction-bound: the run
// bookkeeping cost more than it saved at ~1 edge per run.)
// ---------------------------------------------------------------------------------------------------
struct RgcnEdgeArgs {
    const int32_t* nbr; const int32_t* eid; const float* norm; const float* norm_user;
    const int32_t* type; const int32_t* pos; int64_t n;
    const float* table; int64_t ldt;
    const float* W; int R, Fg, Fo; int transpose;
    float* H; int ldh;
};

constexpr int kEdgeChunk = 256;   // consecutive type-major edges per warp (8 x 32)

template <int FG4, int FO4>
__global__ void __launch_bounds__(256) k_rgcn_edge(const RgcnEdgeArgs a) {
    constexpr int FO = 4 * FO4;
    __shared__ float4 wsm[8][16][FO4];                    // per warp: W'_r of the warp's current type
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const int64_t wid = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t e0 = wid * kEdgeChunk;
    int cur = -1;
    for (int it = 0; it < kEdgeChunk / 32; ++it) {       // warp-uniform
        const int64_t e = e0 + it * 32 + lane;
        const bool live = e < a.n;
        if (e0 + it * 32 >= a.n) break;
        int u = 0, t = -1, p = 0;
        float w = 0.f;
        if (live) {
            u = __ldcs(a.nbr + e);
            t = __ldcs(a.type + e);
            p = __ldcs(a.pos + e);
            w = a.norm_user ? __ldg(a.norm_user + __ldcs(a.eid + e)) : __ldcs(a.norm + e);
        }
        float x[4 * FG4];
        if (live) {
            const float* xr = a.table + (int64_t)u * a.ldt;
#pragma unroll
            for (int q = 0; q < FG4; ++q) {
                const float4 v = ldg4(xr + 4 * q);
                x[4 * q] = v.x * w; x[4 * q + 1] = v.y * w; x[4 * q + 2] = v.z * w; x[4 * q + 3] = v.w * w;
            }
        } else {
#pragma unroll
            for (int i = 0; i < 4 * FG4; ++i) x[i] = 0.f;
        }
#pragma unroll
        for (int i = 0; i < 4 * FG4; ++i)
            if (i >= a.Fg) x[i] = 0.f;                    // the row padding is never read into a result
        // the warp's edges are type-major: stage W'_t of lane 0's type in the warp's slot when it changes
        const int t0 = __shfl_sync(0xffffffffu, t, 0);
        if (t0 != cur && t0 >= 0) {
            cur = t0;
            __syncwarp();
            float* ws = reinterpret_cast<float*>(wsm[wib]);
            for (int idx = lane; idx < 16 * FO; idx += 32) {
                const int i = idx / FO, j = idx % FO;
                float wv = 0.f;
                if (i < a.Fg && j < a.Fo)
                    wv = a.transpose ? __ldg(a.W + ((int64_t)t0 * a.Fo + j) * a.Fg + i)
                                     : __ldg(a.W + ((int64_t)t0 * a.Fg + i) * a.Fo + j);
                ws[idx] = wv;
            }
            __syncwarp();
        }
        float4 acc[FO4];
#pragma unroll
        for (int j4 = 0; j4 < FO4; ++j4) acc[j4] = make_float4(0.f, 0.f, 0.f, 0.f);
        if (t == cur) {                                   // the common case: broadcast reads of the warp's slot
#pragma unroll
            for (int i = 0; i < 4 * FG4; ++i) {
                if (i < a.Fg) {
#pragma unroll
                    for (int j4 = 0; j4 < FO4; ++j4) {
                        const float4 wv = wsm[wib][i][j4];
                        acc[j4].x = fmaf(x[i], wv.x, acc[j4].x);
                        acc[j4].y = fmaf(x[i], wv.y, acc[j4].y);
                        acc[j4].z = fmaf(x[i], wv.z, acc[j4].z);
                        acc[j4].w = fmaf(x[i], wv.w, acc[j4].w);
                    }
                }
            }
        } else if (live) {                                // a type boundary inside the warp: W_t from global
            for (int i = 0; i < a.Fg; ++i)
#pragma unroll
                for (int j4 = 0; j4 < FO4; ++j4) {
                    float wv[4];
#pragma unroll
                    for (int k = 0; k < 4; ++k) {
                        const int j = 4 * j4 + k;
                        wv[k] = j >= a.Fo ? 0.f
                              : a.transpose ? __ldg(a.W + ((int64_t)t * a.Fo + j) * a.Fg + i)
                                            : __ldg(a.W + ((int64_t)t * a.Fg + i) * a.Fo + j);
                    }
                    acc[j4].x = fmaf(x[i], wv[0], acc[j4].x);
                    acc[j4].y = fmaf(x[i], wv[1], acc[j4].y);
                    acc[j4].z = fmaf(x[i], wv[2], acc[j4].z);
                    acc[j4].w = fmaf(x[i], wv[3], acc[j4].w);
                }
        }
        if (live) {
            float4* ho = reinterpret_cast<float4*>(a.H + (int64_t)p * a.ldh);
#pragma unroll
            for (int j4 = 0; j4 < FO4; ++j4) ho[j4] = acc[j4];   // padding columns are 0
        }
    }
}

struct RgcnRowsumArgs {
    const int32_t* perm; const int32_t* row_off; int64_t row_begin, row_end, vbase;
    const float* H; int ldh; int Fo;
    float* out; int64_t ldo;
    const float* bias; int act; int transpose; const float* Yact;
};

// phase 2: LR lanes per row (float4 chunk c of the Fo outputs).  WARP: rows with many slots get a warp each (SL =
// 32/LR slot lanes, slots dealt round-robin, fixed xor-tree merge); else 32/LR rows per warp.  One row per group and
// launch (oversubscribed grid): the row's offsets, vertex id and activation input are loaded up front, the slot
// loads are 4-deep predicated batches.
template <int LR, bool WARP>
__global__ void __launch_bounds__(256) k_rgcn_rowsum(const RgcnRowsumArgs a) {
    constexpr int SL = WARP ? 32 / LR : 1;
    constexpr int RPW = WARP ? 1 : 32 / LR;
    const int lane = threadIdx.x & 31;
    const int c = lane % LR, sl = WARP ? lane / LR : 0;
    const int64_t wid = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t row = a.row_begin + wid * RPW + (WARP ? 0 : lane / LR);
    const bool live = row < a.row_end;
    float acc[4] = {0.f, 0.f, 0.f, 0.f};
    int64_t v = 0;
    float yv[4] = {0.f, 0.f, 0.f, 0.f};
    const bool store = live && sl == 0 && 4 * c < a.Fo;
    if (live) {
        const int b = __ldg(a.row_off + row), e = __ldg(a.row_off + row + 1);
        v = (int64_t)__ldg(a.perm + row) - a.vbase;
        if (store && a.transpose && a.Yact) {
            const float* py = a.Yact + v * a.ldo + 4 * c;
#pragma unroll
            for (int q = 0; q < 4; ++q) yv[q] = 4 * c + q < a.Fo ? __ldg(py + q) : 0.f;
        }
        if (4 * c < a.ldh) {
            for (int k = b + sl; k < e; k += 4 * SL) {        // 4 predicated loads in flight per lane
                float4 x[4];
#pragma unroll
                for (int j = 0; j < 4; ++j)
                    x[j] = k + j * SL < e ? ldg4(a.H + (int64_t)(k + j * SL) * a.ldh + 4 * c) : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
                for (int j = 0; j < 4; ++j) { acc[0] += x[j].x; acc[1] += x[j].y; acc[2] += x[j].z; acc[3] += x[j].w; }
            }
        }
    }
    if (WARP) {
#pragma unroll
        for (int o = LR; o < 32; o <<= 1)
#pragma unroll
            for (int q = 0; q < 4; ++q) acc[q] += __shfl_xor_sync(0xffffffffu, acc[q], o);
    }
    if (!store) return;
    float* po = a.out + v * a.ldo + 4 * c;
    float z[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        const int j = 4 * c + q;
        z[q] = acc[q];
        if (!a.transpose) z[q] = act_apply(a.act, z[q] + ((a.bias && j < a.Fo) ? __ldg(a.bias + j) : 0.f));
        else if (a.Yact) z[q] *= act_grad_from_y(a.act, yv[q]);
    }
    if (4 * c + 4 <= a.Fo && (a.ldo & 3) == 0 && aligned16(a.out)) {
        *reinterpret_cast<float4*>(po) = make_float4(z[0], z[1], z[2], z[3]);      // whole sectors, one store
    } else {
#pragma unroll
        for (int q = 0; q < 4; ++q)
            if (4 * c + q < a.Fo) po[q] = z[q];
    }
}

static size_t em_ws_bytes(const EdgeMajor& em, int64_t Fo) {
    return em.n > 0 ? (size_t)em.n * (size_t)((Fo + 3) & ~3) * sizeof(float) + 256 : 0;
}

// Opt-in (SEASTAR_RGCN_TWOPHASE=1): measured on the AM shape (r2, profiles/r2/README.md) the lane-per-edge product
// kernel is latency-bound at one 1024-thread CTA per SM (W staged whole: 136 KB) and the per-row sums of hub rows
// (degree up to ~7,000) leave a long tail, so the two phases together (0.6 + 0.6 ms for layer 1) lose to the one-pass
// kernel (0.74 ms); the one-pass kernel stays the default.
static bool two_phase(const EdgeMajor& em, int R, int64_t Fg, int64_t Fo) {
    (void)R;
    const char* on = getenv("SEASTAR_RGCN_TWOPHASE");
    return on != nullptr && on[0] == '1' && em.n > 0 && Fg <= 16 && Fo <= 16;
}

// a = the one-pass argument block (table, W, epilogue); x = the index set (rows, offsets, buckets)
static seastar_status launch_two_phase(const IndexSet& x, const EdgeMajor& em, const RgcnRowArgs& a, void* ws,
                                       cudaStream_t s) {
    RgcnEdgeArgs p{};
    p.nbr = em.nbr; p.eid = em.eid; p.norm = em.norm; p.norm_user = a.norm_user;
    p.type = em.type; p.pos = em.pos; p.n = em.n;
    p.table = a.table; p.ldt = a.ldt; p.W = a.W; p.R = a.R; p.Fg = a.Fg; p.Fo = a.Fo; p.transpose = a.transpose;
    p.H = static_cast<float*>(ws); p.ldh = (a.Fo + 3) & ~3;
    const int64_t warps = (em.n + kEdgeChunk - 1) / kEdgeChunk;
    const int64_t blocks = (warps + 7) / 8;
    auto go = [&](auto kern) -> seastar_status {
        launch_k(kern, dim3((unsigned)blocks), dim3(256), 0, s, p);
        return check_launch("k_rgcn_edge");
    };
    const int fg4 = (a.Fg + 3) / 4, fo4 = (a.Fo + 3) / 4;
#define RGCN_EDGE_FO(G4)                                                   \
    switch (fo4) {                                                         \
        case 1: SS_TRY(go(k_rgcn_edge<G4, 1>)); break;                     \
        case 2: SS_TRY(go(k_rgcn_edge<G4, 2>)); break;                     \
        case 3: SS_TRY(go(k_rgcn_edge<G4, 3>)); break;                     \
        default: SS_TRY(go(k_rgcn_edge<G4, 4>)); break;                    \
    }
    switch (fg4) {
        case 1: RGCN_EDGE_FO(1) break;
        case 2: RGCN_EDGE_FO(2) break;
        case 3: RGCN_EDGE_FO(3) break;
        default: RGCN_EDGE_FO(4) break;
    }
#undef RGCN_EDGE_FO
    RgcnRowsumArgs q{};
    q.perm = x.perm; q.row_off = x.off; q.vbase = a.vbase;
    q.H = p.H; q.ldh = p.ldh; q.Fo = a.Fo; q.out = a.out; q.ldo = a.ldo;
    q.bias = a.bias; q.act = a.act; q.transpose = a.transpose; q.Yact = a.Yact;
    const int64_t split = x.bucket_rows[1];                  // rows with degree >= 32: a warp per row
    const int LR = (a.Fo + 3) / 4;
    auto sum = [&](auto lr_tag) -> seastar_status {
        constexpr int L = decltype(lr_tag)::value;
        if (split > 0) {
            RgcnRowsumArgs h = q;
            h.row_begin = 0; h.row_end = split;
            k_rgcn_rowsum<L, true><<<(unsigned)((split + 7) / 8), 256, 0, s>>>(h);
            SS_TRY(check_launch("k_rgcn_rowsum(warp)"));
        }
        if (x.n_rows > split) {
            RgcnRowsumArgs l = q;
            l.row_begin = split; l.row_end = x.n_rows;
            const int64_t rows_per_block = 8 * (32 / L);
            k_rgcn_rowsum<L, false><<<(unsigned)((x.n_rows - split + rows_per_block - 1) / rows_per_block), 256, 0, s>>>(l);
            SS_TRY(check_launch("k_rgcn_rowsum"));
        }
        return SEASTAR_OK;
    };
    switch (LR) {
        case 1: return sum(std::integral_constant<int, 1>{});
        case 2: return sum(std::integral_constant<int, 2>{});
        default: return sum(std::integral_constant<int, 4>{});
    }
}

struct RgcnDwArgs {
    const int32_t* src; const int32_t* eid; const float* norm; const float* norm_user; const int32_t* dst;
    const int32_t* run_off; const int32_t* run_dst; const int32_t* task_run;
    int64_t n_tasks;
    const float* X; int64_t ldx; const float* dA; int64_t ldd;
    int Fin, Fout;
    float* part;
};

// one CTA (8 warps) per task of one type: warp w owns the contiguous edge slice w/8 of the task (its first
// run found by binary search over run_off; a run cut at a slice border contributes its two parts
// g1 (x) dA_v + g2 (x) dA_v, which is exact), keeps its dW_r partial (Fin x Fout, NPL per lane) in registers,
// and the 8 partials are summed in warp order into part[task] (deterministic, no atomics).
template <int L, int NPL>
__global__ void __launch_bounds__(256) k_rgcn_dw(const RgcnDwArgs a) {
    constexpr int S = 32 / L, WARPS = 8;
    __shared__ float sg[WARPS][64];
    __shared__ float sd[WARPS][64];
    extern __shared__ float red[];                 // [WARPS][Fin * Fout]
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int slot = lane / L, c = lane % L;
    const int Cg = (a.Fin + 3) / 4;
    const int FF = a.Fin * a.Fout;
    for (int64_t t = blockIdx.x; t < a.n_tasks; t += gridDim.x) {
        float acc[NPL];
#pragma unroll
        for (int i = 0; i < NPL; ++i) acc[i] = 0.f;
        const int r0 = __ldg(a.task_run + t), r1 = __ldg(a.task_run + t + 1);
        const int es = __ldg(a.run_off + r0), ee = __ldg(a.run_off + r1);
        const int64_t n = ee - es;
        const int k0 = es + (int)(n * w / WARPS), k1 = es + (int)(n * (w + 1) / WARPS);
        if (k0 < k1) {
            int lo = r0, hi = r1 - 1;                  // last run with run_off <= k0
            while (lo < hi) {
                const int mid = (lo + hi + 1) >> 1;
                if (__ldg(a.run_off + mid) <= k0) lo = mid; else hi = mid - 1;
            }
            int run = lo;
            for (int k = k0; k < k1; ++run) {
                const int rend = min(__ldg(a.run_off + run + 1), k1);
                const int64_t v = __ldg(a.run_dst + run);
                float g[4] = {0.f, 0.f, 0.f, 0.f};
                for (int kk = k + slot; kk < rend; kk += S) {
                    if (c < Cg) {
                        const int u = __ldg(a.src + kk);
                        const float wgt = a.norm_user ? __ldg(a.norm_user + __ldg(a.eid + kk)) : __ldg(a.norm + kk);
                        const float4 x = ldg4(a.X + (int64_t)u * a.ldx + 4 * c);
                        g[0] = fmaf(wgt, x.x, g[0]); g[1] = fmaf(wgt, x.y, g[1]);
                        g[2] = fmaf(wgt, x.z, g[2]); g[3] = fmaf(wgt, x.w, g[3]);
                    }
                }
#pragma unroll
                for (int o = L; o < 32; o <<= 1)
#pragma unroll
                    for (int q = 0; q < 4; ++q) g[q] += __shfl_xor_sync(0xffffffffu, g[q], o);
                if (slot == 0 && c < Cg)
#pragma unroll
                    for (int q = 0; q < 4; ++q)
                        if (4 * c + q < a.Fin) sg[w][4 * c + q] = g[q];
                for (int j = lane; j < a.Fout; j += 32) sd[w][j] = __ldg(a.dA + v * a.ldd + j);
                __syncwarp();
#pragma unroll
                for (int i = 0; i < NPL; ++i) {
                    const int e = lane + 32 * i;
                    if (e < FF) acc[i] = fmaf(sg[w][e / a.Fout], sd[w][e % a.Fout], acc[i]);
                }
                __syncwarp();
                k = rend;
            }
        }
#pragma unroll
        for (int i = 0; i < NPL; ++i) {
            const int e = lane + 32 * i;
            if (e < FF) red[w * FF + e] = acc[i];
        }
        __syncthreads();
        for (int e = threadIdx.x; e < FF; e += blockDim.x) {
            float x = red[e];
#pragma unroll
            for (int w2 = 1; w2 < WARPS; ++w2) x += red[w2 * FF + e];
            a.part[t * FF + e] = x;
        }
        __syncthreads();
    }
}

// Narrow layers (F_in <= 16, F_out <= 16: every R-GCN config): a group of L lanes (lane c holds input
// features 2c, 2c+1) owns a contiguous edge slice of the task -- 8 warps x 32/L groups per task -- and keeps
// its dW_r partial (2 x 4*FO4 per lane) in registers.  The slice is walked in batches of L edges: lane c loads edge
// k + c's (source, norm, destination) -- one coalesced round trip per batch -- then the batch's L source rows are
// gathered back to back, and the dA row of every destination that opens a run inside the batch is fetched by the
// lane owning that edge into the group's shared-memory slot (one round trip, only for run starts).  Runs are
// maximal stretches of equal destination inside a task (a task never crosses a type), so no run offsets or binary
// search are needed (the r1 kernel's per-slice binary search and one-edge-at-a-time walk were latency-bound); a run
// cut at a slice border contributes its two parts (exact by linearity).  Groups are merged by a fixed xor tree,
// warps in warp order (deterministic).
template <int L, int FO4>
__global__ void __launch_bounds__(256) k_rgcn_dw_g(const RgcnDwArgs a) {
    constexpr int S = 32 / L, WARPS = 8, G = WARPS * S, FO = 4 * FO4;
    extern __shared__ float red[];                 // [WARPS][Fin * Fout]
    __shared__ float4 dsm[G][L + 1][FO4];          // dA rows of the batch's run starts; [L] = the open run's row
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int slot = lane / L, c = lane % L;
    const int grp = w * S + slot;
    const int FF = a.Fin * a.Fout;
    const unsigned gmask = (L == 32) ? 0xffffffffu : (((1u << L) - 1u) << (slot * L));
    for (int64_t t = blockIdx.x; t < a.n_tasks; t += gridDim.x) {
        float acc[2][FO];
#pragma unroll
        for (int i = 0; i < 2; ++i)
#pragma unroll
            for (int j = 0; j < FO; ++j) acc[i][j] = 0.f;
        const int r0 = __ldg(a.task_run + t), r1 = __ldg(a.task_run + t + 1);
        const int es = __ldg(a.run_off + r0), ee = __ldg(a.run_off + r1);
        const int64_t n = ee - es;
        const int k0 = es + (int)(n * grp / G), k1 = es + (int)(n * (grp + 1) / G);
        int cur = -1;                                  // destination of the open run (-1: none)
        float g[2] = {0.f, 0.f};
        auto flush = [&]() {                           // acc += g (x) dA[open run]
#pragma unroll
            for (int j4 = 0; j4 < FO4; ++j4) {
                const float4 d = dsm[grp][L][j4];      // broadcast within the group
#pragma unroll
                for (int i = 0; i < 2; ++i) {
                    acc[i][4 * j4] = fmaf(g[i], d.x, acc[i][4 * j4]);
                    acc[i][4 * j4 + 1] = fmaf(g[i], d.y, acc[i][4 * j4 + 1]);
                    acc[i][4 * j4 + 2] = fmaf(g[i], d.z, acc[i][4 * j4 + 2]);
                    acc[i][4 * j4 + 3] = fmaf(g[i], d.w, acc[i][4 * j4 + 3]);
                }
            }
        };
        for (int k = k0; k < k1; k += L) {             // trip counts differ by <= 1 across the warp's groups
            const int nb = min(L, k1 - k);
            int u_l = 0, d_l = -1;
            float n_l = 0.f;
            if (c < nb) {
                u_l = __ldg(a.src + k + c);
                d_l = __ldg(a.dst + k + c);
                n_l = a.norm_user ? __ldg(a.norm_user + __ldg(a.eid + k + c)) : __ldg(a.norm + k + c);
            }
            // does edge k + c open a run (its destination differs from the previous edge's)?
            const int d_prev = __shfl_up_sync(gmask, d_l, 1, L);
            const bool starts = c < nb && d_l != (c == 0 ? cur : d_prev);
            if (starts) {
                const float* dp = a.dA + (int64_t)d_l * a.ldd;
#pragma unroll
                for (int j4 = 0; j4 < FO4; ++j4) {
                    float4 d4 = ldg4(dp + 4 * j4);
                    if (4 * j4 + 0 >= a.Fout) d4.x = 0.f;   // the row padding is never read into a result
                    if (4 * j4 + 1 >= a.Fout) d4.y = 0.f;
                    if (4 * j4 + 2 >= a.Fout) d4.z = 0.f;
                    if (4 * j4 + 3 >= a.Fout) d4.w = 0.f;
                    dsm[grp][c][j4] = d4;
                }
            }
            float2 x[L];
#pragma unroll
            for (int j = 0; j < L; ++j) {
                const int u = __shfl_sync(gmask, u_l, j, L);
                x[j] = (j < nb && 2 * c < a.Fin) ? __ldg(reinterpret_cast<const float2*>(a.X + (int64_t)u * a.ldx + 2 * c))
                                                 : make_float2(0.f, 0.f);
                if (2 * c + 1 >= a.Fin) x[j].y = 0.f;
            }
            // group-local vote: the warp's groups may run one batch apart (slice lengths differ by <= 1 edge)
            const unsigned st = (__ballot_sync(gmask, starts) >> (slot * L)) & ((L == 32) ? 0xffffffffu : ((1u << L) - 1u));
            __syncwarp(gmask);
#pragma unroll
            for (int j = 0; j < L; ++j) {
                if (j < nb) {                          // group-uniform
                    if ((st >> j) & 1u) {              // edge k + j opens a new run
                        if (cur >= 0) flush();
                        g[0] = g[1] = 0.f;
                        cur = __shfl_sync(gmask, d_l, j, L);
                        __syncwarp(gmask);             // flush's reads of the open row before it is replaced
                        for (int j4 = c; j4 < FO4; j4 += L) dsm[grp][L][j4] = dsm[grp][j][j4];
                        __syncwarp(gmask);
                    }
                    const float wj = __shfl_sync(gmask, n_l, j, L);
                    g[0] = fmaf(wj, x[j].x, g[0]);
                    g[1] = fmaf(wj, x[j].y, g[1]);
                }
            }
            __syncwarp(gmask);                          // the batch slots are rewritten by the next batch
        }
        if (cur >= 0) flush();
#pragma unroll
        for (int o = L; o < 32; o <<= 1)
#pragma unroll
            for (int i = 0; i < 2; ++i)
#pragma unroll
                for (int j = 0; j < FO; ++j) acc[i][j] += __shfl_xor_sync(0xffffffffu, acc[i][j], o);
        if (slot == 0)
#pragma unroll
            for (int i = 0; i < 2; ++i)
#pragma unroll
                for (int j = 0; j < FO; ++j)
                    if (2 * c + i < a.Fin && j < a.Fout) red[w * FF + (2 * c + i) * a.Fout + j] = acc[i][j];
        __syncthreads();
        for (int e = threadIdx.x; e < FF; e += blockDim.x) {
            float x = red[e];
#pragma unroll
            for (int w2 = 1; w2 < WARPS; ++w2) x += red[w2 * FF + e];
            a.part[t * FF + e] = x;
        }
        __syncthreads();
    }
}

__global__ void __launch_bounds__(256) k_seg_reduce_cols(const float* __restrict__ part,
                                                          const int32_t* __restrict__ seg_off, int width,
                                                          float* __restrict__ out) {
    __shared__ double red[8][32];
    const int sgi = blockIdx.y, lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int e = blockIdx.x * 32 + lane;
    const int t0 = __ldg(seg_off + sgi), t1 = __ldg(seg_off + sgi + 1);
    double x = 0.0;
    if (e < width) {
#pragma unroll 4
        for (int t = t0 + w; t < t1; t += 8) x += (double)__ldg(part + (int64_t)t * width + e);
    }
    red[w][lane] = x;
    __syncthreads();
    if (w == 0 && e < width) {
        double y = red[0][lane];
#pragma unroll
        for (int k = 1; k < 8; ++k) y += red[k][lane];
        out[(int64_t)sgi * width + e] = (float)y;
    }
}

void seg_reduce_cols(const float* part, const int32_t* seg_off, int nseg, int width, float* out, cudaStream_t s) {
    if (nseg <= 0 || width <= 0) return;
    k_seg_reduce_cols<<<dim3((unsigned)((width + 31) / 32), (unsigned)nseg), 256, 0, s>>>(part, seg_off, width, out);
}

// BS: 1024-thread CTAs for the narrow (L <= 4, <= 64 registers) row kernels, so that a W table too large for two
// CTAs per SM (AM: 133 x 16 x 16 fp32 = 136 KB) still leaves 32 warps per SM to hide the gather latency
template <int L, int RL, int WPR = 1, int BS = (WPR == 1 && L <= 4 ? 1024 : 512)>
static seastar_status launch_rows(const RgcnRowArgs& a, size_t smem, cudaStream_t s) {
    if (a.row_end <= a.row_begin) return SEASTAR_OK;
    // per call (the attribute is per device): a host-side setting, cheap next to the launch
    SS_CUDA(cudaFuncSetAttribute(k_rgcn_rows<L, RL, WPR, BS>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 227 * 1024 - (int)sizeof(float) * 64 * WPR));
    int per_sm = 0;
    SS_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_rgcn_rows<L, RL, WPR, BS>, BS, smem));
    if (per_sm < 1) {
        set_error("rgcn: W (%zu bytes) does not fit in shared memory", smem);
        return SEASTAR_ERR_UNSUPPORTED;
    }
    const int64_t groups = a.row_end - a.row_begin;
    int64_t blocks = (int64_t)per_sm * num_sms();
    const int gpb = WPR > 1 ? 1 : BS / RL;
    const int64_t need = (groups + gpb - 1) / gpb;
    if (blocks > need) blocks = need;
    launch_k(k_rgcn_rows<L, RL, WPR, BS>, dim3((unsigned)blocks), dim3(BS), smem, s, a);
    return check_launch("k_rgcn_rows");
}

template <int L>
static seastar_status launch_buckets(const IndexSet& x, RgcnRowArgs a, size_t smem, cudaStream_t s) {
    const int64_t hub = x.bucket_rows[0];     // degree >= 1024: a 16- or 32-warp CTA per row
    const int64_t split = x.bucket_rows[1];   // rows with degree >= 32 get a warp with 32/L slots
    RgcnRowArgs hb = a, hi = a, lo = a;
    hb.row_begin = 0; hb.row_end = hub;
    hi.row_begin = hub; hi.row_end = split;
    lo.row_begin = split; lo.row_end = x.n_rows;
    constexpr int WH = L <= 4 ? 32 : 16;     // hub rows: one CTA of WH warps (registers allow 1024 threads at L <= 4)
    SS_TRY((launch_rows<L, 32, WH, 32 * WH>(hb, smem, s)));
    SS_TRY((launch_rows<L, 32>(hi, smem, s)));
#ifndef RGCN_RLO
#define RGCN_RLO 4   // lanes per low-degree row (>= L): A/B knob for tools/build_variant.sh
#endif
    constexpr int RLo = L < RGCN_RLO ? RGCN_RLO : L;
    return launch_rows<L, RLo>(lo, smem, s);
}

static seastar_status launch_rows_L(const IndexSet& x, RgcnRowArgs a, cudaStream_t s) {
    const int Cm = ((a.Fg > a.Fo ? a.Fg : a.Fo) + 3) / 4;
    a.wstride = (int)w_stride(a.R, a.Fg, (a.Fo + 3) & ~3);
    const size_t smem = (size_t)a.R * a.wstride * sizeof(float);
    switch (pow2_ceil(Cm)) {
        case 1: return launch_buckets<1>(x, a, smem, s);
        case 2: return launch_buckets<2>(x, a, smem, s);
        case 4: return launch_buckets<4>(x, a, smem, s);
        case 8: return launch_buckets<8>(x, a, smem, s);
        default: return launch_buckets<16>(x, a, smem, s);
    }
}

// the edge-balanced tile path (rgcn_tile.cu) from the one-pass argument block
static RgcnTileArgs tile_args(const IndexSet& x, const RgcnRowArgs& a) {
    RgcnTileArgs t{};
    t.perm = x.perm; t.off = x.off; t.nbr = a.nbr; t.typ = a.typ; t.norm = a.norm; t.eid = a.eid;
    t.norm_user = a.norm_user; t.tile_row = x.tile_row; t.n_rows = x.n_rows; t.n_edges = x.n_edges; t.vbase = a.vbase;
    t.table = a.table; t.ldt = a.ldt; t.W = a.W; t.R = a.R; t.Fg = a.Fg; t.Fo = a.Fo; t.transpose = a.transpose;
    t.out = a.out; t.ldo = a.ldo; t.bias = a.bias; t.act = a.act; t.Yact = a.Yact;
    return t;
}

static bool use_tile(const EdgeMajor& em, const IndexSet& x, int R, int64_t Fg, int64_t Fo) {
    return x.tile_row != nullptr && !two_phase(em, R, Fg, Fo) && rgcn_tile_ok(R, Fg, Fo);
}

}  // namespace seastar

using namespace seastar;

extern "C" {

size_t seastar_rgcn_fwd_workspace(seastar_graph g, int64_t F_in, int64_t F_out) {
    if (!g) return 0;
    if (two_phase(g->fem, g->R, F_in, F_out)) return em_ws_bytes(g->fem, F_out);
    return use_tile(g->fem, g->fwd, g->R, F_in, F_out) ? rgcn_tile_ws_bytes(g->fwd.n_edges) : 0;
}

seastar_status seastar_rgcn_fwd(seastar_graph g, const float* X_all, int64_t F_in, int64_t ldx, const float* W,
                                int64_t F_out, const float* norm_user, const float* bias, seastar_act act,
                                float* Y_loc, int64_t ldy, void* workspace, size_t ws_bytes, seastar_stream stream) {
    SS_ARG(g && X_all && W && Y_loc, "rgcn_fwd: NULL argument");
    SS_ARG(F_in >= 1 && F_in <= 64 && F_out >= 1 && F_out <= 64, "rgcn_fwd: need 1 <= F_in, F_out <= 64");
    SS_ARG(ldx >= F_in && ldx % 4 == 0 && aligned16(X_all), "rgcn_fwd: X_all needs ldx %% 4 == 0 and 16B alignment");
    SS_ARG(ldy >= F_out, "rgcn_fwd: bad ldy");
    SS_ARG(g->fwd.type != nullptr || g->R == 1, "rgcn_fwd: graph has no edge types");
    SS_ARG(norm_user || g->fwd.norm, "rgcn_fwd: pass norm_user or create the graph with SEASTAR_GRAPH_RGCN_NORM");
    SS_ARG(act >= SEASTAR_ACT_NONE && act <= SEASTAR_ACT_SIGMOID, "rgcn_fwd: bad activation");
    SS_ARG(g->fwd.type != nullptr, "rgcn_fwd: graph was created without etypes");
    SS_TRY(check_device());
    RgcnRowArgs a{};
    a.perm = g->fwd.perm; a.off = g->fwd.off; a.nbr = g->fwd.nbr; a.typ = g->fwd.type;
    a.norm = g->fwd.norm; a.eid = g->fwd.eid; a.norm_user = norm_user;
    a.vbase = g->row_begin;
    a.table = X_all; a.ldt = ldx; a.W = W; a.R = g->R; a.Fg = (int)F_in; a.Fo = (int)F_out; a.transpose = 0;
    a.out = Y_loc; a.ldo = ldy; a.bias = bias; a.act = act;
    const size_t need = seastar_rgcn_fwd_workspace(g, F_in, F_out);
    SS_ARG(need == 0 || (workspace && ws_bytes >= need), "rgcn_fwd: workspace too small (%zu < %zu bytes)", ws_bytes,
           need);
    ScopedL2Window win(X_all, (size_t)g->N * ldx * sizeof(float));
    if (two_phase(g->fem, g->R, F_in, F_out)) return launch_two_phase(g->fwd, g->fem, a, workspace, to_stream(stream));
    if (use_tile(g->fem, g->fwd, g->R, F_in, F_out))
        return rgcn_tile_launch(tile_args(g->fwd, a), g->fwd.bucket_rows[2], workspace, to_stream(stream));
    return launch_rows_L(g->fwd, a, to_stream(stream));
}

size_t seastar_rgcn_bwd_workspace(seastar_graph g, int64_t F_in, int64_t F_out) {
    if (!g) return 0;
    // dW task partials and (two-phase dX) the per-segment products: used one after the other
    const size_t dw = (size_t)(g->tm.n_tasks + 1) * (size_t)(F_in * F_out) * sizeof(float) + 256;
    const size_t dx = two_phase(g->rem, g->R, F_out, F_in)  ? em_ws_bytes(g->rem, F_in)
                      : use_tile(g->rem, g->rev, g->R, F_out, F_in) ? rgcn_tile_ws_bytes(g->rev.n_edges)
                                                            : 0;
    return dw > dx ? dw : dx;
}

seastar_status seastar_rgcn_bwd(seastar_graph g, const float* X_all, int64_t F_in, int64_t ldx, const float* dA_all,
                                int64_t F_out, int64_t ldd, const float* W, const float* norm_user,
                                const float* Yact_loc, seastar_act act, float* dX_loc, float* dW, void* workspace,
                                size_t ws_bytes, seastar_stream stream) {
    SS_ARG(g && X_all && dA_all && W, "rgcn_bwd: NULL argument");
    SS_ARG(act >= SEASTAR_ACT_NONE && act <= SEASTAR_ACT_SIGMOID, "rgcn_bwd: bad activation");
    SS_ARG(dX_loc || dW, "rgcn_bwd: nothing to compute");
    SS_ARG(F_in >= 1 && F_in <= 64 && F_out >= 1 && F_out <= 64, "rgcn_bwd: need 1 <= F_in, F_out <= 64");
    SS_ARG(F_in * F_out <= 32 * 32, "rgcn_bwd: F_in * F_out <= 1024 required for the register dW path");
    SS_ARG(ldx >= F_in && ldx % 4 == 0 && aligned16(X_all), "rgcn_bwd: X_all needs ldx %% 4 == 0, 16B alignment");
    SS_ARG(ldd >= F_out && ldd % 4 == 0 && aligned16(dA_all), "rgcn_bwd: dA_all needs ldd %% 4 == 0, 16B alignment");
    SS_ARG(g->fwd.type != nullptr, "rgcn_bwd: graph was created without etypes");
    SS_ARG(norm_user || g->fwd.norm, "rgcn_bwd: pass norm_user or create the graph with SEASTAR_GRAPH_RGCN_NORM");
    SS_ARG(!dW || (workspace && ws_bytes >= seastar_rgcn_bwd_workspace(g, F_in, F_out)),
           "rgcn_bwd: workspace too small");
    // argument checks stay before any launch: the two-phase dX needs the workspace as well
    SS_ARG(!dX_loc || (!two_phase(g->rem, g->R, F_out, F_in) && !use_tile(g->rem, g->rev, g->R, F_out, F_in)) ||
           (workspace && ws_bytes >= seastar_rgcn_bwd_workspace(g, F_in, F_out)), "rgcn_bwd: workspace too small");
    SS_TRY(check_device());
    cudaStream_t s = to_stream(stream);
    if (dX_loc) {
        RgcnRowArgs a{};
        a.perm = g->rev.perm; a.off = g->rev.off; a.nbr = g->rev.nbr; a.typ = g->rev.type;
        a.norm = g->rev.norm; a.eid = g->rev.eid; a.norm_user = norm_user;
        a.vbase = g->row_begin;
        a.table = dA_all; a.ldt = ldd; a.W = W; a.R = g->R; a.Fg = (int)F_out; a.Fo = (int)F_in; a.transpose = 1;
        a.out = dX_loc; a.ldo = ldx; a.bias = nullptr; a.act = act; a.Yact = Yact_loc;
        ScopedL2Window win(dA_all, (size_t)g->N * ldd * sizeof(float));
        if (two_phase(g->rem, g->R, F_out, F_in)) {
            SS_ARG(workspace && ws_bytes >= seastar_rgcn_bwd_workspace(g, F_in, F_out), "rgcn_bwd: workspace too small");
            SS_TRY(launch_two_phase(g->rev, g->rem, a, workspace, s));
        } else if (use_tile(g->rem, g->rev, g->R, F_out, F_in)) {
            SS_TRY(rgcn_tile_launch(tile_args(g->rev, a), g->rev.bucket_rows[2], workspace, s));
        } else {
            SS_TRY(launch_rows_L(g->rev, a, s));
        }
    }
    if (dW) {
        const int FF = (int)(F_in * F_out);
        if (g->tm.n_tasks > 0) {
            RgcnDwArgs d{};
            d.src = g->tm.src; d.eid = g->tm.eid; d.norm = g->tm.norm; d.norm_user = norm_user; d.dst = g->tm.dst;
            d.run_off = g->tm.run_off; d.run_dst = g->tm.run_dst; d.task_run = g->tm.task_run;
            d.n_tasks = g->tm.n_tasks;
            d.X = X_all; d.ldx = ldx; d.dA = dA_all; d.ldd = ldd; d.Fin = (int)F_in; d.Fout = (int)F_out;
            d.part = static_cast<float*>(workspace);
            ScopedL2Window win(X_all, (size_t)g->N * ldx * sizeof(float));
            const int Cg = (int)((F_in + 3) / 4);
            const int L = pow2_ceil(Cg);
            const int npl = pow2_ceil((FF + 31) / 32);
            const size_t smem_r = (size_t)8 * FF * sizeof(float);
            int64_t blocks = 0;
#define RGCN_DW(LL, NN)                                                                                  \
    do {                                                                                                 \
        int per_sm = 0;                                                                                  \
        SS_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_rgcn_dw<LL, NN>, 256, smem_r)); \
        blocks = (int64_t)(per_sm > 0 ? per_sm : 1) * num_sms();                                         \
        if (blocks > g->tm.n_tasks) blocks = g->tm.n_tasks;                                              \
        launch_k(k_rgcn_dw<LL, NN>, dim3((unsigned)blocks), dim3(256), smem_r, s, d);                    \
    } while (0)
#define RGCN_DW_L(LL)                                                   \
    switch (npl) {                                                      \
        case 1: RGCN_DW(LL, 1); break;                                  \
        case 2: RGCN_DW(LL, 2); break;                                  \
        case 4: RGCN_DW(LL, 4); break;                                  \
        case 8: RGCN_DW(LL, 8); break;                                  \
        case 16: RGCN_DW(LL, 16); break;                                \
        default: RGCN_DW(LL, 32); break;                                \
    }
#define RGCN_DWG(LL, F4)                                                                                \
    do {                                                                                                  \
        int per_sm = 0;                                                                                   \
        SS_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_rgcn_dw_g<LL, F4>, 256, smem_r)); \
        blocks = (int64_t)(per_sm > 0 ? per_sm : 1) * num_sms();                                          \
        if (blocks > g->tm.n_tasks) blocks = g->tm.n_tasks;                                               \
        launch_k(k_rgcn_dw_g<LL, F4>, dim3((unsigned)blocks), dim3(256), smem_r, s, d);                   \
    } while (0)
#define RGCN_DWG_L(LL)                   \
    switch ((F_out + 3) / 4) {           \
        case 1: RGCN_DWG(LL, 1); break;  \
        case 2: RGCN_DWG(LL, 2); break;  \
        case 3: RGCN_DWG(LL, 3); break;  \
        default: RGCN_DWG(LL, 4); break; \
    }
            const char* dwg = getenv("SEASTAR_RGCN_DWG");   // A/B: the r2 register-walk dW kernel
            if (F_in <= 16 && F_out <= 16 && !(dwg && dwg[0] == '1')) {
                RgcnDwTileArgs t{};
                t.src = d.src; t.dst = d.dst; t.eid = d.eid; t.norm = d.norm; t.norm_user = d.norm_user;
                t.run_off = d.run_off; t.task_run = d.task_run; t.n_tasks = d.n_tasks;
                t.X = d.X; t.ldx = d.ldx; t.dA = d.dA; t.ldd = d.ldd; t.Fin = d.Fin; t.Fout = d.Fout; t.part = d.part;
                SS_TRY(rgcn_dw_tile_launch(t, s));
            } else if (F_in <= 16 && F_out <= 16) {
                switch (pow2_ceil((int)((F_in + 1) / 2))) {   // lanes per group: 2 input features per lane
                    case 1: RGCN_DWG_L(1); break;
                    case 2: RGCN_DWG_L(2); break;
                    case 4: RGCN_DWG_L(4); break;
                    default: RGCN_DWG_L(8); break;
                }
            } else {
                switch (L) {
                    case 1: RGCN_DW_L(1); break;
                    case 2: RGCN_DW_L(2); break;
                    case 4: RGCN_DW_L(4); break;
                    case 8: RGCN_DW_L(8); break;
                    default: RGCN_DW_L(16); break;
                }
            }
#undef RGCN_DWG_L
#undef RGCN_DWG
#undef RGCN_DW_L
#undef RGCN_DW
            SS_TRY(check_launch("k_rgcn_dw"));
            seg_reduce_cols(static_cast<float*>(workspace), g->tm.type_task, g->R, FF, dW, s);
            SS_TRY(check_launch("k_seg_reduce_cols"));
        } else {
            SS_CUDA(cudaMemsetAsync(dW, 0, sizeof(float) * (size_t)g->R * FF, s));
        }
    }
    return SEASTAR_OK;
}

}  // extern "C"
