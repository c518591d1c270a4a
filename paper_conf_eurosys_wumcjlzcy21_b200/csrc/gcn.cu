// gcn.cu -- a5 / a8: fused GCN / APPNP aggregation, forward on the degree-sorted CSR and backward
// on the degree-sorted reverse CSR (Fig. 1 L85-L93, Fig. 3, Alg. 1,
// §6.3.2 "vertex-parallel edge-sequential", §6.3.4).
//
// B200 mapping (prior art: the paper's FAT groups, §6.3.1; not copied):
//   * a row's features are split into L "chunk lanes" of VEC floats (128-bit loads when VEC = 4);
//   * a row group of RL lanes (RL = 32: one warp per row; RL = L: several rows per warp for the
//     low-degree bucket) owns one destination row; its S = RL / L edge slots walk the row's edges,
//     RL edge ids at a time (one coalesced 32-bit load per lane, broadcast by shuffles), with UB
//     gathers in flight per lane;
//   * partial sums stay in registers and are merged by a fixed xor-shuffle tree: no atomics, no
//     shared memory, bitwise deterministic;
//   * rows are degree-sorted (hubs first, similar degrees share a warp), the grid is oversubscribed
//     and the block scheduler's id order provides the dynamic load balance of §6.3.3 (L437-L453);
//   * the epilogue (norm, APPNP mix, bias, activation, next-layer pre-scaling / activation
//     derivative) is fused so each output row is written once.
#include <algorithm>

#include "common.cuh"

namespace seastar {

struct AggArgs {
    const int32_t* perm;   // row -> vertex id
    const int32_t* off;    // row offsets
    const int32_t* nbr;    // neighbour ids per edge
    int64_t row_begin;     // first row of this launch (bucket)
    int64_t row_end;       // one past the last row of this launch
    int64_t vbase;         // owned vertex base (row_begin of the partition)
    const float* table;    // gathered rows [N, ld]
    int64_t ld;
    int F;
    int bwd;               // 0: forward epilogue, 1: backward epilogue
    const float* rscale;   // per-vertex scale [n_loc] (dst_norm fwd / src_norm bwd) or null
    float gscale;          // global scale (1 fwd, APPNP (1-alpha) bwd)
    // forward
    const float* H0; float alpha; const float* bias; int act; float* Y; const float* out_scale; float* Ys;
    // backward
    const float* Yact; float* dA; const float* post_scale; float* dP;
    // NEXT-3 edge dropout (deid == nullptr: off): edge k's message is scaled by drop_mult(key, eid[k])
    const int32_t* deid; uint64_t dseed; const int32_t* dstep; uint32_t dsite, dthr; float dscale;
    int64_t nlong;         // WPR > 1 launches: blocks [0, nlong) are long rows (a CTA each), the rest 8 warp-rows
    // NEXT-1 split phases over a LocalSplit (phase 0: whole rows, no split): phase 1 sums each row's owned-neighbour
    // edges from tloc (the rank's own rows, ld ldloc) into part (ld ldp, no epilogue) while the all-gather of the
    // table runs; phase 2 sums the remaining edges from the gathered table, adds part, and runs the epilogue
    int phase; const int32_t* lcnt; const float* tloc; int64_t ldloc; float* part; int64_t ldp;
};

// minimum resident blocks.  Measured on Reddit (r1/r2): with one index chunk per iteration, forcing 6 blocks (40
// registers) sped the plain-sum sweep at F = 32 / 64 (1.12 / 2.00 -> 1.01 / 1.88 ms) but slowed the GCN training
// aggregation (0.68 -> 0.73 ms).  r2 (second session): two index chunks per iteration for warp rows (AGG_NB4 = 2,
// 64 edges' gathers in flight per warp: the kernel is bound by bytes in flight, long-scoreboard stalls) at 4 blocks
// per SM (64 registers): GCN aggregation 0.68 -> 0.61 ms; NB = 2 at the compiler's 66 registers 0.79 ms, at 5 blocks
// (spills) 0.78 ms, NB = 3 at 4 blocks 0.78 ms (tools/ab_reddit.sh)
#ifndef AGG_MB
#define AGG_MB 4
#endif
// (applied to the two-chunk warp-row instances only: the other classes keep the compiler's choice -- at 4 blocks the
// APPNP propagation on the Physics shape lost 10 %)
#define AGG_BOUNDS __launch_bounds__(256, (AGG_MB > 0 && L >= 4 && NB >= 2) ? AGG_MB : 1)
// WPR > 1 (RL = 32, WPR = the block's warps): the launch's first a.nlong blocks each own one long row (long_rows():
// degree above a quarter of one SM's share of the launch) -- warp w walks the w-th contiguous slice of the row's
// edges, and the warps' partial sums are added in warp order through shared memory before warp 0 runs the epilogue
// (deterministic) -- and every later block owns 8 rows, a warp each ("CTA + Warp").  One
// launch for both classes: a separate hub launch cost more (kernel boundary) than it saved on the Reddit shape.
// PH: NEXT-1 split phase (0: whole rows; 1 / 2: see AggArgs) as a template parameter -- a runtime phase cost the
// whole-row kernel 14 registers (48 -> 62) and its occupancy (r2 sweep: 0.67 -> 0.81 ms at F = 16 on Reddit)
template <int VEC, int L, int RL, int NB, bool DROP = false, int WPR = 1, int PH = 0>
__global__ void AGG_BOUNDS k_aggregate(const AggArgs a) {
    static_assert(WPR == 1 || RL == 32, "hub rows take whole warps");
    constexpr int S = RL / L;                    // edge slots per row group
#ifdef GCN_UB_FIXED
    constexpr int UB = GCN_UB_FIXED < 32 / L ? GCN_UB_FIXED : 32 / L;
#else
    constexpr int UB = (L < 4 ? L : 4);          // gathers per lane per index chunk and batch
#endif
    const int lane = threadIdx.x & 31;
    const int gl = lane % RL;                    // lane within the row group
    const int slot = gl / L;
    const int c = gl % L;
    const unsigned gmask = (RL == 32) ? 0xffffffffu : (((1u << RL) - 1u) << ((lane / RL) * RL));
    const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int wib = threadIdx.x >> 5;            // warp in block (the slice index when WPR > 1)
    const bool hubblk = WPR > 1 && (int64_t)blockIdx.x < a.nlong;      // block-uniform
    const int64_t row = hubblk ? a.row_begin + blockIdx.x
                      : WPR > 1 ? a.row_begin + a.nlong + ((int64_t)blockIdx.x - a.nlong) * (blockDim.x >> 5) + wib
                                : a.row_begin + warp * (32 / RL) + lane / RL;
    const bool valid = row < a.row_end;
    int beg = valid ? __ldg(a.off + row) : 0;
    int end = valid ? __ldg(a.off + row + 1) : 0;
    if (PH != 0 && valid) {                      // NEXT-1: owned-neighbour edges lead every split row
        const int lc = __ldg(a.lcnt + row);
        if (PH == 1) end = beg + lc; else beg += lc;
    }
    const float* tab = PH == 1 ? a.tloc - a.vbase * a.ldloc : a.table;   // phase 1: the rank's own rows
    const int64_t tld = PH == 1 ? a.ldloc : a.ld;
    if (hubblk) {
        const int64_t len = end - beg;
        const int b0 = beg + (int)(len * wib / WPR);
        end = beg + (int)(len * (wib + 1) / WPR);
        beg = b0;
    }
    const int64_t v = valid ? (int64_t)__ldg(a.perm + row) - a.vbase : 0;
    const int C = (a.F + VEC - 1) / VEC;
    const uint64_t dkey = DROP ? drop_key(a.dseed, a.dsite, a.dstep) : 0ull;

    for (int cb = 0; cb < C; cb += L) {
        const int chunk = cb + c;
        const bool active = chunk < C;
        const int64_t col = (int64_t)chunk * VEC;
        float acc[VEC];
#pragma unroll
        for (int i = 0; i < VEC; ++i) acc[i] = 0.f;

        // NB chunks of RL edge ids per iteration, software-pipelined: the next iteration's index
        // loads are issued before this iteration's gathers, so an iteration costs one memory round
        // trip (the gathers) instead of two (index load, then the dependent gathers)
        int nxt[NB];
#pragma unroll
        for (int h = 0; h < NB; ++h) nxt[h] = (gl < end - beg - h * RL) ? __ldcs(a.nbr + beg + h * RL + gl) : 0;
        for (int base = beg; base < end; base += NB * RL) {
            int n[NB], my[NB];
#pragma unroll
            for (int h = 0; h < NB; ++h) {
                n[h] = max(0, min(RL, end - base - h * RL));
                my[h] = nxt[h];
                const int nb = base + (NB + h) * RL;
                nxt[h] = (gl < end - nb) ? __ldcs(a.nbr + nb + gl) : 0;
            }
#pragma unroll
            for (int j0 = 0; j0 < L; j0 += UB) {
                if (j0 * S >= n[0]) break;
                float val[NB][UB][VEC];
#pragma unroll
                for (int h = 0; h < NB; ++h)
#pragma unroll
                    for (int jj = 0; jj < UB; ++jj) {
                        const int k = (j0 + jj) * S + slot;
                        const int u = __shfl_sync(gmask, my[h], k & (RL - 1), RL);
                        if (k < n[h] && active) {
                            load_vec<VEC>(tab + (int64_t)u * tld + col, val[h][jj]);
                            if (DROP) {
                                const float w = drop_mult(dkey, (uint64_t)__ldg(a.deid + base + h * RL + k), a.dthr,
                                                          a.dscale);
#pragma unroll
                                for (int i = 0; i < VEC; ++i) val[h][jj][i] *= w;
                            }
                        } else {
#pragma unroll
                            for (int i = 0; i < VEC; ++i) val[h][jj][i] = 0.f;
                        }
                    }
#pragma unroll
                for (int h = 0; h < NB; ++h)
#pragma unroll
                    for (int jj = 0; jj < UB; ++jj)
#pragma unroll
                        for (int i = 0; i < VEC; ++i) acc[i] += val[h][jj][i];
            }
        }
        // merge the S edge slots (fixed tree)
#pragma unroll
        for (int o = L; o < RL; o <<= 1)
#pragma unroll
            for (int i = 0; i < VEC; ++i) acc[i] += __shfl_xor_sync(gmask, acc[i], o, RL);
        if (hubblk) {                                // merge the warps' slices in warp order
            __shared__ float red[WPR > 1 ? WPR : 1][32][VEC];
            if (slot == 0)
#pragma unroll
                for (int i = 0; i < VEC; ++i) red[wib][c][i] = acc[i];
            __syncthreads();
            if (wib == 0 && slot == 0) {
#pragma unroll
                for (int i = 0; i < VEC; ++i) {
                    float t = red[0][c][i];
                    for (int w2 = 1; w2 < WPR; ++w2) t += red[w2][c][i];
                    acc[i] = t;
                }
            }
            __syncthreads();
            if (wib != 0) continue;
        }

        if (!valid || slot != 0 || !active) continue;
        if (PH == 1) {                               // partial row sum, finished by phase 2
            float* pp = a.part + v * a.ldp + col;
            if (col + VEC <= a.F) store_vec<VEC>(pp, acc);
            else for (int i = 0; i < VEC && col + i < a.F; ++i) pp[i] = acc[i];
            continue;
        }
        if (PH == 2) {
            const float* pp = a.part + v * a.ldp + col;
#pragma unroll
            for (int i = 0; i < VEC; ++i)
                if (col + i < a.F) acc[i] += pp[i];
        }
        const float rs = (a.rscale ? __ldg(a.rscale + v) : 1.f) * a.gscale;
        float out[VEC], out2[VEC];
        if (!a.bwd) {
            const float os = a.out_scale ? __ldg(a.out_scale + v) : 1.f;
#pragma unroll
            for (int i = 0; i < VEC; ++i) {
                float z = acc[i] * rs;
                const int64_t cc = col + i;
                if (cc < a.F) {
                    if (a.H0) z = (1.f - a.alpha) * z + a.alpha * __ldg(a.H0 + v * a.ld + cc);
                    if (a.bias) z += __ldg(a.bias + cc);
                }
                z = act_apply(a.act, z);
                out[i] = z;
                out2[i] = os * z;
            }
            float* y = a.Y + v * a.ld + col;
            float* ys = a.Ys ? a.Ys + v * a.ld + col : nullptr;
            if (col + VEC <= a.F) {
                store_vec<VEC>(y, out);
                if (ys) store_vec<VEC>(ys, out2);
            } else {
                for (int i = 0; i < VEC && col + i < a.F; ++i) {
                    y[i] = out[i];
                    if (ys) ys[i] = out2[i];
                }
            }
        } else {
            const float ps = a.post_scale ? __ldg(a.post_scale + v) : 1.f;
#pragma unroll
            for (int i = 0; i < VEC; ++i) {
                float g = acc[i] * rs;
                if (a.Yact && col + i < a.F) g *= act_grad_from_y(a.act, __ldg(a.Yact + v * a.ld + col + i));
                out[i] = g;
                out2[i] = ps * g;
            }
            float* da = a.dA ? a.dA + v * a.ld + col : nullptr;
            float* dp = a.dP ? a.dP + v * a.ld + col : nullptr;
            if (col + VEC <= a.F) {
                if (da) store_vec<VEC>(da, out);
                if (dp) store_vec<VEC>(dp, out2);
            } else {
                for (int i = 0; i < VEC && col + i < a.F; ++i) {
                    if (da) da[i] = out[i];
                    if (dp) dp[i] = out2[i];
                }
            }
        }
    }
}

constexpr int kHubWarps = 8;       // warps per hub row (degree >= 1024: >= 128 edges per warp)
#ifndef AGG_NB4
#define AGG_NB4 2                  // index chunks per iteration for warp rows with L >= 4 (see AGG_MB)
#endif

template <int VEC, int L, int PH>
static void launch_rl_ph(AggArgs a, bool warp_rows, cudaStream_t s, bool hub) {
    const int64_t rows = a.row_end - a.row_begin;
    if (rows <= 0) return;
    constexpr int threads = 256;
    if (hub) {                                   // long rows (a CTA each) + warp rows in one launch
        static_assert(32 * kHubWarps == threads, "hub CTAs are the launch's 256-thread blocks");
        constexpr int NBW = L >= 4 ? AGG_NB4 : 4 / L;
        const unsigned grid = (unsigned)(a.nlong + (rows - a.nlong + kHubWarps - 1) / kHubWarps);
        if (a.deid) launch_k(k_aggregate<VEC, L, 32, NBW, true, kHubWarps, PH>, dim3(grid), dim3(threads), 0, s, a);
        else launch_k(k_aggregate<VEC, L, 32, NBW, false, kHubWarps, PH>, dim3(grid), dim3(threads), 0, s, a);
        return;
    }
    if (warp_rows) {
        const int64_t blocks = (rows + (threads / 32) - 1) / (threads / 32);
        // NB = 1: measured on Reddit F=16, NB=2 (66 regs) is 18% slower than NB=1 (48 regs): occupancy
        // buys more memory-level parallelism than deeper per-lane batches
        // narrow rows (L < 4 chunk lanes, F <= 8) take 4/L index chunks per iteration so every lane still has
        // 4 gathers in flight: F = 8 0.75 -> 0.50 ms, F = 1..4 0.54 -> 0.46 ms on Reddit (tools/ab_gcn.sh)
        constexpr int NBW = L >= 4 ? AGG_NB4 : 4 / L;
        if (a.deid) launch_k(k_aggregate<VEC, L, 32, NBW, true, 1, PH>, dim3((unsigned)blocks), dim3(threads), 0, s, a);
        else launch_k(k_aggregate<VEC, L, 32, NBW, false, 1, PH>, dim3((unsigned)blocks), dim3(threads), 0, s, a);
    } else {
        constexpr int RL = L < 4 ? 4 : L;   // at least 4 lanes per row group keeps index loads useful
        const int64_t per_block = threads / RL;
        const int64_t blocks = (rows + per_block - 1) / per_block;
        if (a.deid) launch_k(k_aggregate<VEC, L, RL, 1, true, 1, PH>, dim3((unsigned)blocks), dim3(threads), 0, s, a);
        else launch_k(k_aggregate<VEC, L, RL, 1, false, 1, PH>, dim3((unsigned)blocks), dim3(threads), 0, s, a);
    }
}

template <int VEC, int L>
static void launch_rl(AggArgs a, bool warp_rows, cudaStream_t s, bool hub = false) {
    switch (a.phase) {
        case 1: launch_rl_ph<VEC, L, 1>(a, warp_rows, s, hub); break;
        case 2: launch_rl_ph<VEC, L, 2>(a, warp_rows, s, hub); break;
        default: launch_rl_ph<VEC, L, 0>(a, warp_rows, s, hub); break;
    }
}

template <int VEC>
static void launch_vec(AggArgs a, int L, bool warp_rows, cudaStream_t s, bool hub = false) {
    switch (L) {
        case 1: launch_rl<VEC, 1>(a, warp_rows, s, hub); break;
        case 2: launch_rl<VEC, 2>(a, warp_rows, s, hub); break;
        case 4: launch_rl<VEC, 4>(a, warp_rows, s, hub); break;
        case 8: launch_rl<VEC, 8>(a, warp_rows, s, hub); break;
        case 16: launch_rl<VEC, 16>(a, warp_rows, s, hub); break;
        default: launch_rl<VEC, 32>(a, warp_rows, s, hub); break;
    }
}

// launch over the two degree classes of an index set: rows with degree >= 32 get a warp each,
// the rest (incl. empty rows, which still need their epilogue) get sub-warp row groups; sp: the local-first split
// of x (NEXT-1 phases 1 / 2) or nullptr
seastar_status launch_aggregate(const IndexSet& x, AggArgs a, bool vec4, cudaStream_t s,
                                const LocalSplit* sp = nullptr) {
    const int VEC = vec4 ? 4 : 1;
    const int C = (a.F + VEC - 1) / VEC;
    const int L = C >= 32 ? 32 : pow2_ceil(C);
    const int64_t split = x.bucket_rows[1];   // # rows with degree >= 32
    a.perm = x.perm;
    a.off = x.off;
    a.nbr = sp ? sp->nbr : x.nbr;
    a.lcnt = sp ? sp->lcnt : nullptr;
    AggArgs hi = a, lo = a;
    hi.row_begin = 0; hi.row_end = split;
    hi.nlong = std::min<int64_t>(long_rows(x), split);     // long rows lead the degree-sorted order
    lo.row_begin = split; lo.row_end = x.n_rows;
    lo.nlong = 0;
    if (vec4) {
        launch_vec<4>(hi, L, true, s, hi.nlong > 0);
        launch_vec<4>(lo, L, L >= 32, s);
    } else {
        launch_vec<1>(hi, L, true, s, hi.nlong > 0);
        launch_vec<1>(lo, L, L >= 32, s);
    }
    return check_launch("k_aggregate");
}

}  // namespace seastar

using namespace seastar;

extern "C" {

seastar_status seastar_gcn_fwd(seastar_graph g, const float* T_all, int64_t F, int64_t ld, const float* dst_norm,
                               const float* bias, seastar_act act, float alpha, const float* H0_loc, float* Y_loc,
                               const float* out_scale, float* Ys_loc, const seastar_dropout_spec* edge_drop,
                               seastar_stream stream) {
    SS_ARG(g != nullptr, "gcn_fwd: graph is NULL");
    SS_ARG(F >= 1 && ld >= F, "gcn_fwd: need 1 <= F <= ld (F=%lld, ld=%lld)", (long long)F, (long long)ld);
    SS_ARG(T_all != nullptr && Y_loc != nullptr, "gcn_fwd: T_all and Y_loc are required");
    SS_ARG(!Ys_loc || out_scale, "gcn_fwd: Ys_loc requires out_scale");
    SS_ARG(act >= SEASTAR_ACT_NONE && act <= SEASTAR_ACT_SIGMOID, "gcn_fwd: bad activation %d", (int)act);
    SS_ARG((void*)T_all != (void*)Y_loc, "gcn_fwd: output aliases the gathered table");
    SS_TRY(check_device());
    AggArgs a{};
    a.vbase = g->row_begin;
    a.table = T_all; a.ld = ld; a.F = (int)F; a.bwd = 0;
    a.rscale = dst_norm; a.gscale = 1.f;
    a.H0 = H0_loc; a.alpha = alpha; a.bias = bias; a.act = act; a.Y = Y_loc; a.out_scale = out_scale; a.Ys = Ys_loc;
    SS_ARG(!edge_drop || (edge_drop->p >= 0.f && edge_drop->p < 1.f), "gcn_fwd: need 0 <= edge_drop->p < 1");
    set_drop(a, edge_drop, g->fwd.eid);
    bool vec4 = (ld % 4 == 0) && aligned16(T_all) && aligned16(Y_loc) && (!H0_loc || aligned16(H0_loc)) &&
                (!Ys_loc || aligned16(Ys_loc));
    return launch_aggregate(g->fwd, a, vec4, to_stream(stream));
}

seastar_status seastar_gcn_bwd(seastar_graph g, const float* dP_all, int64_t F, int64_t ld, const float* src_norm,
                               float scale, const float* Yact_loc, seastar_act act, const float* post_scale,
                               float* dA_loc, float* dP_loc, const seastar_dropout_spec* edge_drop,
                               seastar_stream stream) {
    SS_ARG(g != nullptr, "gcn_bwd: graph is NULL");
    SS_ARG(F >= 1 && ld >= F, "gcn_bwd: need 1 <= F <= ld");
    SS_ARG(dP_all != nullptr, "gcn_bwd: dP_all is NULL");
    SS_ARG(dA_loc || dP_loc, "gcn_bwd: need dA_loc and/or dP_loc");
    SS_ARG(act >= SEASTAR_ACT_NONE && act <= SEASTAR_ACT_SIGMOID, "gcn_bwd: bad activation %d", (int)act);
    SS_ARG((void*)dP_all != (void*)dA_loc && (void*)dP_all != (void*)dP_loc, "gcn_bwd: output aliases the input");
    SS_TRY(check_device());
    AggArgs a{};
    a.vbase = g->row_begin;
    a.table = dP_all; a.ld = ld; a.F = (int)F; a.bwd = 1;
    a.rscale = src_norm; a.gscale = scale;
    a.Yact = Yact_loc; a.act = act; a.dA = dA_loc; a.post_scale = post_scale; a.dP = dP_loc;
    SS_ARG(!edge_drop || (edge_drop->p >= 0.f && edge_drop->p < 1.f), "gcn_bwd: need 0 <= edge_drop->p < 1");
    set_drop(a, edge_drop, g->rev.eid);
    bool vec4 = (ld % 4 == 0) && aligned16(dP_all) && (!dA_loc || aligned16(dA_loc)) && (!dP_loc || aligned16(dP_loc)) &&
                (!Yact_loc || aligned16(Yact_loc));
    return launch_aggregate(g->rev, a, vec4, to_stream(stream));
}

// NEXT-1: the partitioned aggregation in two phases around the all-gather (seastar.h)
seastar_status seastar_gcn_fwd_split(seastar_graph g, int32_t phase, const float* T_loc, int64_t ldloc,
                                     const float* T_all, int64_t F, int64_t ld, const float* dst_norm,
                                     const float* bias, seastar_act act, float alpha, const float* H0_loc,
                                     float* Y_loc, const float* out_scale, float* Ys_loc, float* part, int64_t ldp,
                                     const seastar_dropout_spec* edge_drop, seastar_stream stream) {
    SS_ARG(g != nullptr, "gcn_fwd_split: graph is NULL");
    SS_ARG(g->partitioned, "gcn_fwd_split: the graph is not row-partitioned (use seastar_gcn_fwd)");
    SS_ARG(phase == 1 || phase == 2, "gcn_fwd_split: phase must be 1 or 2");
    SS_ARG(F >= 1 && ld >= F && ldp >= F, "gcn_fwd_split: bad sizes");
    SS_ARG(part != nullptr, "gcn_fwd_split: part is NULL");
    SS_ARG(phase == 2 || (T_loc && ldloc >= F), "gcn_fwd_split: phase 1 needs T_loc (ldloc >= F)");
    SS_ARG(phase == 1 || (T_all && Y_loc), "gcn_fwd_split: phase 2 needs T_all and Y_loc");
    SS_ARG(!Ys_loc || out_scale, "gcn_fwd_split: Ys_loc requires out_scale");
    SS_ARG(act >= SEASTAR_ACT_NONE && act <= SEASTAR_ACT_SIGMOID, "gcn_fwd_split: bad activation %d", (int)act);
    SS_ARG(!edge_drop || (edge_drop->p >= 0.f && edge_drop->p < 1.f), "gcn_fwd_split: need 0 <= edge_drop->p < 1");
    SS_TRY(check_device());
    AggArgs a{};
    a.vbase = g->row_begin;
    a.table = T_all; a.ld = ld; a.F = (int)F; a.bwd = 0;
    a.rscale = dst_norm; a.gscale = 1.f;
    a.H0 = H0_loc; a.alpha = alpha; a.bias = bias; a.act = act; a.Y = Y_loc; a.out_scale = out_scale; a.Ys = Ys_loc;
    a.phase = phase; a.tloc = T_loc; a.ldloc = ldloc; a.part = part; a.ldp = ldp;
    set_drop(a, edge_drop, g->fsplit.eid);
    const bool vec4 = (ld % 4 == 0) && (ldp % 4 == 0) && aligned16(part) &&
                      (phase == 2 ? aligned16(T_all) && aligned16(Y_loc) && (!H0_loc || aligned16(H0_loc)) &&
                                        (!Ys_loc || aligned16(Ys_loc))
                                  : (ldloc % 4 == 0) && aligned16(T_loc));
    return launch_aggregate(g->fwd, a, vec4, to_stream(stream), &g->fsplit);
}

seastar_status seastar_gcn_bwd_split(seastar_graph g, int32_t phase, const float* dP_loc_in, int64_t ldloc,
                                     const float* dP_all, int64_t F, int64_t ld, const float* src_norm, float scale,
                                     const float* Yact_loc, seastar_act act, const float* post_scale, float* dA_loc,
                                     float* dP_loc, float* part, int64_t ldp, const seastar_dropout_spec* edge_drop,
                                     seastar_stream stream) {
    SS_ARG(g != nullptr, "gcn_bwd_split: graph is NULL");
    SS_ARG(g->partitioned, "gcn_bwd_split: the graph is not row-partitioned (use seastar_gcn_bwd)");
    SS_ARG(phase == 1 || phase == 2, "gcn_bwd_split: phase must be 1 or 2");
    SS_ARG(F >= 1 && ld >= F && ldp >= F, "gcn_bwd_split: bad sizes");
    SS_ARG(part != nullptr, "gcn_bwd_split: part is NULL");
    SS_ARG(phase == 2 || (dP_loc_in && ldloc >= F), "gcn_bwd_split: phase 1 needs dP_loc_in (ldloc >= F)");
    SS_ARG(phase == 1 || (dP_all && (dA_loc || dP_loc)), "gcn_bwd_split: phase 2 needs dP_all and an output");
    SS_ARG(act >= SEASTAR_ACT_NONE && act <= SEASTAR_ACT_SIGMOID, "gcn_bwd_split: bad activation %d", (int)act);
    SS_ARG(!edge_drop || (edge_drop->p >= 0.f && edge_drop->p < 1.f), "gcn_bwd_split: need 0 <= edge_drop->p < 1");
    SS_TRY(check_device());
    AggArgs a{};
    a.vbase = g->row_begin;
    a.table = dP_all; a.ld = ld; a.F = (int)F; a.bwd = 1;
    a.rscale = src_norm; a.gscale = scale;
    a.Yact = Yact_loc; a.act = act; a.dA = dA_loc; a.post_scale = post_scale; a.dP = dP_loc;
    a.phase = phase; a.tloc = dP_loc_in; a.ldloc = ldloc; a.part = part; a.ldp = ldp;
    set_drop(a, edge_drop, g->rsplit.eid);
    const bool vec4 = (ld % 4 == 0) && (ldp % 4 == 0) && aligned16(part) &&
                      (phase == 2 ? aligned16(dP_all) && (!dA_loc || aligned16(dA_loc)) &&
                                        (!dP_loc || aligned16(dP_loc)) && (!Yact_loc || aligned16(Yact_loc))
                                  : (ldloc % 4 == 0) && aligned16(dP_loc_in));
    return launch_aggregate(g->rev, a, vec4, to_stream(stream), &g->rsplit);
}

}  // extern "C"
