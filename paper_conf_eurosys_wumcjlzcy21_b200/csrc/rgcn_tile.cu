// rgcn_tile.cu -- a7 / a10: the R-GCN layer over edge-balanced tiles with a CTA-local type grouping
// (§6.3.5, the hierarchical "sum per type, then over types" aggregation of [53]).
//
// Why a second formulation.  The paper sorts each row's edges by type and detects type changes (L473-L475), so a
// row pushes every (row, type) run through W_r.  On the AM shape (mean in-degree 3, 133 relations) a run is ~1 edge,
// so the one-pass kernel (rgcn.cu, k_rgcn_rows) reads a whole W_r (1 KB) from shared memory per *edge* and stays
// shared-memory bound at ~11 % of HBM.  Here the W_r reads are shared by all edges of one type inside a
// tile instead of inside a row:
//   tile t = the edges [t*CAP, (t+1)*CAP) of the index set in row order (every CTA gets the same number of edges,
//            whatever the degree distribution -- hub rows simply span several tiles);
//   stage  : the tile's gathered rows table[nbr_e] land in shared memory (cp.async, 16 B per lane, all in flight),
//            its (type, norm) records next to them;
//   group  : a counting sort by type in shared memory gives the tile's edges in type-major order (the order inside
//            a type does not matter: every edge's product has its own slot);
//   product: warp w walks a contiguous stretch of the type-major order, each half-warp a contiguous half of it, 4
//            edges per step; lane (j, e) keeps column j of W_r in registers and reloads it only when its half-warp's
//            type changes; per edge the half-warp reads the staged row by broadcast and the message
//            m_e = norm_e * (table[nbr_e] W_r) overwrites the edge's staged row;
//            (warp-aggregated __match_any_sync counters for the sort were measured slower: 0.62 -> 0.68 ms on AM)
//   sum    : each row sums its contiguous message slots in row order (type, eid) and applies the epilogue; a row
//            cut by a tile border leaves its partial sum in the workspace (head: the part of a row that began in an
//            earlier tile; tail: a row that continues into the next tile), and k_rgcn_tile_fix adds a cut row's
//            parts in tile order.
// Deterministic (every sum has a fixed order; the only atomics are the shared-memory counters of the type sort,
// which place edges but never add floats).  Forward: table = X, W'_r = W_r, epilogue act(. + b).  dX (REV CSR):
// table = dA, W'_r = W_r^T, epilogue * act'(Yact).
#include "common.cuh"
#include "rgcn_tile.cuh"

namespace seastar {

namespace {

constexpr int kTileThreads = 256;    // standalone tile kernel (W read through L1/L2)
#ifndef RGCN_TILE_PT
#define RGCN_TILE_PT 512
#endif
constexpr int kTilePThreads = RGCN_TILE_PT;      // persistent tile kernel (one CTA per SM, W resident in smem)
#ifndef RGCN_W_SWIZZLE
#define RGCN_W_SWIZZLE 1
#endif
constexpr bool kRgcnWSwizzle = RGCN_W_SWIZZLE;   // bank-conflict-free W' column reloads (FG4 = 4)

__device__ __forceinline__ void cp_async16(void* smem, const void* gmem) {
    const unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(gmem) : "memory");
}
// 16-byte copy of the first `bytes` bytes, the rest of the 16 zero-filled (the row padding never reaches a result)
__device__ __forceinline__ void cp_async16z(void* smem, const void* gmem, int bytes) {
    const unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(s), "l"(gmem), "r"(bytes) : "memory");
}
__device__ __forceinline__ void cp_async4(void* smem, const void* gmem) {
    const unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;\n" ::"r"(s), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait0() { asm volatile("cp.async.wait_group 0;\n" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() {
    cp_async_commit();
    cp_async_wait0();
}

// one tile's staging area in shared memory
struct TileBuf {
    float4* slot;      // [CAP][SW4] gathered rows, overwritten by the messages
    float* snorm;      // [CAP]
    int32_t* sperm;    // [CAP]     vertex of row r_lo + k
    int32_t* soff;     // [CAP + 4] raw row offsets off[r_lo + k]
    uint16_t* stype;   // [CAP]
};
template <int SW4>
__host__ __device__ constexpr size_t tile_buf_bytes() {
    return (size_t)kRgcnTileEdges * (SW4 * 16 + 4 + 4 + 2) + (kRgcnTileEdges + 4) * 4;
}
template <int SW4>
__device__ __forceinline__ TileBuf carve(uint8_t* p) {
    constexpr int CAP = kRgcnTileEdges;
    TileBuf b;
    b.slot = reinterpret_cast<float4*>(p);
    b.snorm = reinterpret_cast<float*>(b.slot + CAP * SW4);
    b.sperm = reinterpret_cast<int32_t*>(b.snorm + CAP);
    b.soff = b.sperm + CAP;
    b.stype = reinterpret_cast<uint16_t*>(b.soff + CAP + 4);
    return b;
}

struct EdgeRec {
    int u = 0, ty = 0;
    float w = 0.f;
};
__device__ __forceinline__ EdgeRec load_rec(const RgcnTileArgs& a, int64_t e) {
    EdgeRec r;
    r.u = __ldcs(a.nbr + e);
    r.ty = __ldcs(a.typ + e);
    r.w = a.norm_user ? __ldg(a.norm_user + __ldcs(a.eid + e)) : __ldcs(a.norm + e);
    return r;
}
template <int FG4, int SW4>
__device__ __forceinline__ void issue_edge(const RgcnTileArgs& a, const TileBuf& b, int i, const EdgeRec& r) {
    b.stype[i] = (uint16_t)r.ty;
    b.snorm[i] = r.w;
    const float* src = a.table + (int64_t)r.u * a.ldt;
#pragma unroll
    for (int q = 0; q < FG4; ++q) {
        const int bytes = a.Fg - 4 * q >= 4 ? 16 : 4 * (a.Fg - 4 * q);
        cp_async16z(b.slot + i * SW4 + q, src + 4 * q, bytes);
    }
}
__device__ __forceinline__ void issue_rows(const RgcnTileArgs& a, const TileBuf& b, int64_t r_lo, int nr, int tid,
                                           int nt) {
    for (int k = tid; k <= nr; k += nt) {
        cp_async4(b.soff + k, a.off + r_lo + k);
        if (k < nr) cp_async4(b.sperm + k, a.perm + r_lo + k);
    }
}

// epilogue of output chunk c (columns 4c .. 4c+3) of vertex v; yv = the activation inputs (dX with Yact only)
__device__ __forceinline__ void tile_store(const RgcnTileArgs& a, int64_t v, int c, const float (&z)[4],
                                           const float (&yv)[4]) {
    float* po = a.out + v * a.ldo + 4 * c;
    float y[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        const int j = 4 * c + q;
        if (!a.transpose) y[q] = j < a.Fo ? act_apply(a.act, z[q] + (a.bias ? __ldg(a.bias + j) : 0.f)) : 0.f;
        else y[q] = a.Yact ? z[q] * act_grad_from_y(a.act, yv[q]) : z[q];
    }
    if (4 * c + 4 <= a.Fo && (a.ldo & 3) == 0 && aligned16(a.out)) {
        *reinterpret_cast<float4*>(po) = make_float4(y[0], y[1], y[2], y[3]);
    } else {
#pragma unroll
        for (int q = 0; q < 4; ++q)
            if (4 * c + q < a.Fo) po[q] = y[q];
    }
}

__device__ __forceinline__ void load_yact(const RgcnTileArgs& a, int64_t v, int c, float (&yv)[4]) {
#pragma unroll
    for (int q = 0; q < 4; ++q)
        yv[q] = (a.transpose && a.Yact && 4 * c + q < a.Fo) ? __ldg(a.Yact + v * a.ldo + 4 * c + q) : 0.f;
}

// W'_t[k][j] (k < Fg gathered feature, j < Fo output): the forward uses W_t, dX its transpose
__device__ __forceinline__ float w_prime(const RgcnTileArgs& a, int t, int k, int j) {
    return a.transpose ? __ldg(a.W + ((int64_t)t * a.Fo + j) * a.Fg + k) : __ldg(a.W + ((int64_t)t * a.Fg + k) * a.Fo + j);
}

// Steps 2-4 of one staged tile (sort by type, products, row sums).  WS: W' resident in shared memory as
// [R][16][4 FG4] (persistent kernel; else read through L1/L2).
template <int FG4, int FO4, int NT, bool WS>
__device__ __forceinline__ void process_tile(const RgcnTileArgs& a, const TileBuf& b, uint32_t* order, int* hist,
                                             const float* Ws, int64_t tile, int64_t e0, int n, int64_t r_lo, int nr) {
    constexpr int NW = NT / 32;
    constexpr int SW4 = FG4 > FO4 ? FG4 : FO4;
    constexpr unsigned FULL = 0xffffffffu;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    // counting sort by type: counts, exclusive scan, placement (afterwards hist[t] = end of type t's range)
    for (int r = tid; r < a.R; r += NT) hist[r] = 0;
    __syncthreads();
    for (int i = tid; i < n; i += NT) atomicAdd(&hist[b.stype[i]], 1);
    __syncthreads();
    if (warp == 0) {
        int carry = 0;
        for (int q = 0; q < a.R; q += 32) {
            const int v = q + lane < a.R ? hist[q + lane] : 0;
            int x = v;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int y = __shfl_up_sync(FULL, x, o);
                if (lane >= o) x += y;
            }
            if (q + lane < a.R) hist[q + lane] = carry + x - v;
            carry += __shfl_sync(FULL, x, 31);
        }
    }
    __syncthreads();
    for (int i = tid; i < n; i += NT) {
        const int t = b.stype[i];
        order[atomicAdd(&hist[t], 1)] = ((uint32_t)t << 16) | (uint32_t)i;
    }
    __syncthreads();
    // products: lane (j, e) keeps column j of W'_t (all 4 FG4 gathered features) for its half-warp's current type t,
    // reloaded only when the type changes, and computes output j of its half-warp's edges from the staged rows
    // (broadcast reads; four independent FMA chains per edge).  order[] packs (type << 16 | slot).
    {
        constexpr int KP = 4 * FG4;
        const int j = lane & 15, e = lane >> 4;
        const int p0 = n * warp / NW, p1 = n * (warp + 1) / NW;
        float w[KP];
#pragma unroll
        for (int k = 0; k < KP; ++k) w[k] = 0.f;
        int cur = -1;
        auto reload = [&](int t) {
            cur = t;
            if constexpr (WS) {
                const float4* wc = reinterpret_cast<const float4*>(Ws + (t * 16 + j) * KP);
#pragma unroll
                for (int q = 0; q < FG4; ++q) {
                    const float4 v = wc[(FG4 == 4 && kRgcnWSwizzle) ? (q + (j >> 1)) & 3 : q];
                    w[4 * q] = v.x; w[4 * q + 1] = v.y; w[4 * q + 2] = v.z; w[4 * q + 3] = v.w;
                }
            } else {
#pragma unroll
                for (int k = 0; k < KP; ++k) w[k] = (k < a.Fg && j < a.Fo) ? w_prime(a, t, k, j) : 0.f;
            }
        };
        auto dot = [&](const float4 (&x)[FG4]) {
            float m[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
            for (int q = 0; q < FG4; ++q) {                  // padding: x zero-filled, w zero
                m[0] = fmaf(x[q].x, w[4 * q], m[0]);
                m[1] = fmaf(x[q].y, w[4 * q + 1], m[1]);
                m[2] = fmaf(x[q].z, w[4 * q + 2], m[2]);
                m[3] = fmaf(x[q].w, w[4 * q + 3], m[3]);
            }
            return (m[0] + m[1]) + (m[2] + m[3]);
        };
        // each half-warp walks its own contiguous half of the stretch, UE edges per step (their rows' loads all in
        // flight before the FMAs); both halves step together (warp-uniform trip count and branch: a step takes the
        // fast path when every live edge of both halves has its half's current type)
        constexpr int UE = 4;
        const int pm = p0 + (p1 - p0 + 1) / 2;
        const int q0 = e ? pm : p0, q1 = e ? p1 : pm;
        const int steps = (pm - p0 + UE - 1) / UE;           // the first half is the longer one
        for (int st = 0; st < steps; ++st) {                 // warp-uniform trip count
            const int pb = q0 + st * UE;
            uint32_t o[UE];
            float4 x[UE][FG4];
#pragma unroll
            for (int u = 0; u < UE; ++u) {
                o[u] = pb + u < q1 ? order[pb + u] : 0xffffffffu;
                const int i = o[u] != 0xffffffffu ? (int)(o[u] & 0xffffu) : 0;
#pragma unroll
                for (int q = 0; q < FG4; ++q) x[u][q] = b.slot[i * SW4 + q];
            }
            bool same = true;
#pragma unroll
            for (int u = 0; u < UE; ++u) same &= (o[u] == 0xffffffffu) || (int)(o[u] >> 16) == cur;
            float m[UE];
            if (__all_sync(FULL, same)) {                    // warp-uniform
#pragma unroll
                for (int u = 0; u < UE; ++u) m[u] = dot(x[u]);
            } else {
#pragma unroll
                for (int u = 0; u < UE; ++u) {
                    if (o[u] != 0xffffffffu && (int)(o[u] >> 16) != cur) reload((int)(o[u] >> 16));
                    m[u] = dot(x[u]);
                }
            }
            float nrm[UE];
#pragma unroll
            for (int u = 0; u < UE; ++u) nrm[u] = o[u] != 0xffffffffu ? b.snorm[o[u] & 0xffffu] : 0.f;
            __syncwarp();                                    // every lane's reads of its rows before the writes
            if (j < 4 * FO4) {
#pragma unroll
                for (int u = 0; u < UE; ++u)
                    if (o[u] != 0xffffffffu) reinterpret_cast<float*>(b.slot + (o[u] & 0xffffu) * SW4)[j] = m[u] * nrm[u];
            }
        }
    }
    __syncthreads();
    // row sums in row order; rows cut by a tile border leave a partial in the workspace
    const int c = lane & 3;
    auto seg = [&](int k) {
        const int lo = b.soff[k] - (int)e0;              // offsets < 2^31 (validated at graph_create)
        return lo < 0 ? 0 : (lo > n ? n : lo);
    };
    auto finish = [&](int k, const float (&z)[4], const float (&yv)[4]) {
        const bool head = k == 0 && b.soff[0] < e0;
        const bool tail = !head && k == nr - 1 && b.soff[nr] > e0 + n;
        if (!head && !tail) {
            if (c < FO4) tile_store(a, b.sperm[k] - a.vbase, c, z, yv);
        } else if (c < FO4) {
            float* pp = a.part + (tile * 2 + (head ? 0 : 1)) * 16 + 4 * c;
            *reinterpret_cast<float4*>(pp) = make_float4(z[0], z[1], z[2], z[3]);
        }
    };
    if (nr <= 2 * NW) {
        // few (long) rows: a warp per row, 8 slot lanes x 4 chunk lanes, slots dealt round-robin, fixed xor merge
        const int sl = lane >> 2;
        for (int k = warp; k < nr; k += NW) {
            float yv[4];
            load_yact(a, b.sperm[k] - a.vbase, c, yv);
            const int lo = seg(k), en = seg(k + 1);
            float z0[4] = {0.f, 0.f, 0.f, 0.f}, z1[4] = {0.f, 0.f, 0.f, 0.f};
            if (c < FO4) {
                int q = lo + sl;
                for (; q + 8 < en; q += 16) {
                    const float4 v0 = b.slot[q * SW4 + c], v1 = b.slot[(q + 8) * SW4 + c];
                    z0[0] += v0.x; z0[1] += v0.y; z0[2] += v0.z; z0[3] += v0.w;
                    z1[0] += v1.x; z1[1] += v1.y; z1[2] += v1.z; z1[3] += v1.w;
                }
                if (q < en) {
                    const float4 v0 = b.slot[q * SW4 + c];
                    z0[0] += v0.x; z0[1] += v0.y; z0[2] += v0.z; z0[3] += v0.w;
                }
            }
            float z[4];
#pragma unroll
            for (int qq = 0; qq < 4; ++qq) {
                z[qq] = z0[qq] + z1[qq];
#pragma unroll
                for (int o = 4; o < 32; o <<= 1) z[qq] += __shfl_xor_sync(FULL, z[qq], o);
            }
            if (sl == 0) finish(k, z, yv);
        }
    } else {
        // many short rows: 4 chunk lanes per row, 8 rows per warp
        for (int k = warp * 8 + (lane >> 2); k < nr; k += NW * 8) {
            float yv[4];
            load_yact(a, b.sperm[k] - a.vbase, c, yv);
            const int lo = seg(k), en = seg(k + 1);
            float z[4] = {0.f, 0.f, 0.f, 0.f};
            if (c < FO4)
                for (int q = lo; q < en; ++q) {
                    const float4 v = b.slot[q * SW4 + c];
                    z[0] += v.x; z[1] += v.y; z[2] += v.z; z[3] += v.w;
                }
            finish(k, z, yv);
        }
    }
}

}  // namespace

// standalone: one tile per CTA, W' read through L1/L2 (used when W does not fit in shared memory next to the tiles)
template <int FG4, int FO4>
__global__ void __launch_bounds__(kTileThreads) k_rgcn_tile(const RgcnTileArgs a) {
    constexpr int CAP = kRgcnTileEdges, NT = kTileThreads;
    constexpr int SW4 = FG4 > FO4 ? FG4 : FO4;
    extern __shared__ float4 smem[];
    uint8_t* base = reinterpret_cast<uint8_t*>(smem);
    const TileBuf b = carve<SW4>(base);
    uint32_t* order = reinterpret_cast<uint32_t*>(base + tile_buf_bytes<SW4>());
    int* hist = reinterpret_cast<int*>(order + CAP);
    const int tid = threadIdx.x;
    const int64_t tile = blockIdx.x, e0 = tile * CAP;
    const int n = (int)min((int64_t)CAP, a.n_edges - e0);
    const int64_t r_lo = __ldg(a.tile_row + 2 * tile);
    const int nr = (int)(__ldg(a.tile_row + 2 * tile + 1) - r_lo + 1);
    for (int i = tid; i < n; i += NT) issue_edge<FG4, SW4>(a, b, i, load_rec(a, e0 + i));
    issue_rows(a, b, r_lo, nr, tid, NT);
    cp_async_wait_all();
    __syncthreads();
    process_tile<FG4, FO4, NT, false>(a, b, order, hist, nullptr, tile, e0, n, r_lo, nr);
}

// persistent: one CTA of 512 threads per SM, W' = [R][16][4 FG4] staged once in shared memory, two tile buffers: the
// gather of tile t + G (G = grid size) is in flight while tile t is processed, and the edge records of tile t + 2G are
// loaded into registers
template <int FG4, int FO4>
__global__ void __launch_bounds__(kTilePThreads, 1) k_rgcn_tile_p(const RgcnTileArgs a, int64_t n_tiles) {
    constexpr int CAP = kRgcnTileEdges, NT = kTilePThreads;
    constexpr int SW4 = FG4 > FO4 ? FG4 : FO4;
    static_assert(CAP <= NT, "one edge record per thread");
    extern __shared__ float4 smem[];
    uint8_t* base = reinterpret_cast<uint8_t*>(smem);
    const TileBuf buf0 = carve<SW4>(base), buf1 = carve<SW4>(base + tile_buf_bytes<SW4>());
    uint32_t* order = reinterpret_cast<uint32_t*>(base + 2 * tile_buf_bytes<SW4>());
    int* hist = reinterpret_cast<int*>(order + CAP);
    float* Ws = reinterpret_cast<float*>(hist + ((a.R + 3) & ~3));
    const int tid = threadIdx.x;
    const int G = gridDim.x;
    int64_t t = blockIdx.x;
    if (t >= n_tiles) return;
    auto tile_n = [&](int64_t tt) { return (int)min((int64_t)CAP, a.n_edges - tt * CAP); };
    // tile t: records and gather in flight before W is staged
    int2 rng_cur = make_int2(__ldg(a.tile_row + 2 * t), __ldg(a.tile_row + 2 * t + 1));
    if (tid < tile_n(t)) issue_edge<FG4, SW4>(a, buf0, tid, load_rec(a, t * CAP + tid));
    issue_rows(a, buf0, rng_cur.x, rng_cur.y - rng_cur.x + 1, tid, NT);
    cp_async_commit();
    int2 rng_nx = make_int2(0, 0);
    EdgeRec rec_nx;
    if (t + G < n_tiles) {
        rng_nx = make_int2(__ldg(a.tile_row + 2 * (t + G)), __ldg(a.tile_row + 2 * (t + G) + 1));
        if (tid < tile_n(t + G)) rec_nx = load_rec(a, (t + G) * CAP + tid);
    }
    for (int idx = tid; idx < a.R * 16 * 4 * FG4; idx += NT) {      // W'_r as [R][16 (j)][4 FG4 (k)]
        const int k = idx % (4 * FG4), j = (idx / (4 * FG4)) & 15, r = idx / (64 * FG4);
        // FG4 = 4: chunk q of column j sits at chunk (q + j / 2) % 4, so the 8 lanes of a reload's quarter-warp hit 8
        // different 16-byte bank groups (column stride 64 B: unswizzled, lanes j and j + 2 collide)
        const int pk = (FG4 == 4 && kRgcnWSwizzle) ? ((((k >> 2) + (j >> 1)) & 3) << 2) | (k & 3) : k;
        Ws[idx - k + pk] = (j < a.Fo && k < a.Fg) ? w_prime(a, r, k, j) : 0.f;
    }
    for (int it = 0; t < n_tiles; ++it, t += G) {
        const TileBuf& cur = (it & 1) ? buf1 : buf0;
        const TileBuf& nxt = (it & 1) ? buf0 : buf1;
        cp_async_wait0();
        __syncthreads();                                     // tile t landed; the previous tile's processing is done
        const int2 rng_issued = rng_nx;
        if (t + G < n_tiles) {
            if (tid < tile_n(t + G)) issue_edge<FG4, SW4>(a, nxt, tid, rec_nx);
            issue_rows(a, nxt, rng_nx.x, rng_nx.y - rng_nx.x + 1, tid, NT);
            cp_async_commit();
            if (t + 2 * G < n_tiles) {
                const int64_t t2 = t + 2 * G;
                rng_nx = make_int2(__ldg(a.tile_row + 2 * t2), __ldg(a.tile_row + 2 * t2 + 1));
                if (tid < tile_n(t2)) rec_nx = load_rec(a, t2 * CAP + tid);
            }
        }
        process_tile<FG4, FO4, NT, true>(a, cur, order, hist, Ws, t, t * CAP, tile_n(t), rng_cur.x, rng_cur.y - rng_cur.x + 1);
        rng_cur = rng_issued;
    }
}

// rows cut by tile borders (summed over their tiles in tile order) and rows without edges (epilogue of 0)
template <int FO4>
__global__ void __launch_bounds__(256) k_rgcn_tile_fix(const RgcnTileArgs a, int64_t n_tiles, int64_t z0) {
    constexpr int CAP = kRgcnTileEdges;
    const int64_t gid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int c = (int)(gid & 3);
    const int64_t grp = gid >> 2;                          // 4 chunk lanes per tile / per empty row
    float yv[4];
    if (grp < n_tiles - 1) {
        const int64_t t = grp, e1 = (t + 1) * CAP;          // t is not the last tile: e1 < n_edges
        const int64_t row = __ldg(a.tile_row + 2 * t + 1);
        const int64_t beg = __ldg(a.off + row), end = __ldg(a.off + row + 1);
        if (beg >= t * CAP && end > e1 && c < FO4) {        // the row starts in tile t and continues
            const int64_t v = (int64_t)__ldg(a.perm + row) - a.vbase;
            load_yact(a, v, c, yv);
            const float4 p = *reinterpret_cast<const float4*>(a.part + (t * 2 + 1) * 16 + 4 * c);
            float z[4] = {p.x, p.y, p.z, p.w};
            const int64_t tl = (end - 1) / CAP;
            for (int64_t u = t + 1; u <= tl; ++u) {
                const float4 h = *reinterpret_cast<const float4*>(a.part + (u * 2) * 16 + 4 * c);
                z[0] += h.x; z[1] += h.y; z[2] += h.z; z[3] += h.w;
            }
            tile_store(a, v, c, z, yv);
        }
        return;
    }
    const int64_t row = z0 + (grp - (n_tiles > 0 ? n_tiles - 1 : 0));
    if (row < a.n_rows && c < FO4) {
        const int64_t v = (int64_t)__ldg(a.perm + row) - a.vbase;
        const float z[4] = {0.f, 0.f, 0.f, 0.f};
        load_yact(a, v, c, yv);
        tile_store(a, v, c, z, yv);
    }
}

static size_t buf_bytes(int sw4) {
    switch (sw4) {
        case 1: return tile_buf_bytes<1>();
        case 2: return tile_buf_bytes<2>();
        case 3: return tile_buf_bytes<3>();
        default: return tile_buf_bytes<4>();
    }
}
// standalone kernel / persistent kernel dynamic shared memory
static size_t smem_standalone(int R, int sw4) { return buf_bytes(sw4) + kRgcnTileEdges * 4 + (size_t)R * 4; }
static size_t smem_persistent(int R, int Fg, int sw4) {
    return 2 * buf_bytes(sw4) + kRgcnTileEdges * 4 + (size_t)((R + 3) & ~3) * 4 + (size_t)R * 16 * ((Fg + 3) & ~3) * 4;
}
constexpr size_t kSmemCap = 227 * 1024;

bool rgcn_tile_ok(int R, int64_t Fg, int64_t Fo) {
    if (const char* env = getenv("SEASTAR_RGCN_ROWS"))     // A/B: the one-pass row kernel
        if (env[0] == '1') return false;
    if (!(Fg >= 1 && Fg <= 16 && Fo >= 1 && Fo <= 16 && R >= 1 && R <= 65535)) return false;
    const int sw4 = (int)(((Fg > Fo ? Fg : Fo) + 3) / 4);
    return smem_standalone(R, sw4) <= kSmemCap;
}

size_t rgcn_tile_ws_bytes(int64_t n_edges) {
    const int64_t tiles = (n_edges + kRgcnTileEdges - 1) / kRgcnTileEdges;
    return (size_t)(tiles > 0 ? tiles : 1) * 2 * 16 * sizeof(float) + 256;
}

seastar_status rgcn_tile_launch(const RgcnTileArgs& a0, int64_t zero_rows_begin, void* ws, cudaStream_t s) {
    RgcnTileArgs a = a0;
    a.part = static_cast<float*>(ws);
    const int64_t tiles = (a.n_edges + kRgcnTileEdges - 1) / kRgcnTileEdges;
    const int fg4 = (a.Fg + 3) / 4, fo4 = (a.Fo + 3) / 4;
    const int sw4 = fg4 > fo4 ? fg4 : fo4;
    const size_t smem_p = smem_persistent(a.R, a.Fg, sw4), smem_s = smem_standalone(a.R, sw4);
    const char* env = getenv("SEASTAR_RGCN_TILE_STANDALONE");   // A/B: the standalone kernel
    const bool persistent = smem_p <= kSmemCap && !(env && env[0] == '1');
    auto go = [&](auto kern_s, auto kern_p) -> seastar_status {
        if (persistent) {
            SS_CUDA(cudaFuncSetAttribute(kern_p, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_p));
            const int64_t grid = tiles < num_sms() ? tiles : num_sms();
            launch_k(kern_p, dim3((unsigned)grid), dim3(kTilePThreads), smem_p, s, a, tiles);
            return check_launch("k_rgcn_tile_p");
        }
        SS_CUDA(cudaFuncSetAttribute(kern_s, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_s));
        launch_k(kern_s, dim3((unsigned)tiles), dim3(kTileThreads), smem_s, s, a);
        return check_launch("k_rgcn_tile");
    };
    if (tiles > 0) {
#define RGCN_TILE_FO(G4)                                                                  \
    switch (fo4) {                                                                        \
        case 1: SS_TRY(go(k_rgcn_tile<G4, 1>, k_rgcn_tile_p<G4, 1>)); break;              \
        case 2: SS_TRY(go(k_rgcn_tile<G4, 2>, k_rgcn_tile_p<G4, 2>)); break;              \
        case 3: SS_TRY(go(k_rgcn_tile<G4, 3>, k_rgcn_tile_p<G4, 3>)); break;              \
        default: SS_TRY(go(k_rgcn_tile<G4, 4>, k_rgcn_tile_p<G4, 4>)); break;             \
    }
        switch (fg4) {
            case 1: RGCN_TILE_FO(1) break;
            case 2: RGCN_TILE_FO(2) break;
            case 3: RGCN_TILE_FO(3) break;
            default: RGCN_TILE_FO(4) break;
        }
#undef RGCN_TILE_FO
    }
    const int64_t groups = (tiles > 0 ? tiles - 1 : 0) + (a.n_rows - zero_rows_begin);
    if (groups <= 0) return SEASTAR_OK;
    const unsigned blocks = (unsigned)((groups * 4 + 255) / 256);
    switch (fo4) {
        case 1: k_rgcn_tile_fix<1><<<blocks, 256, 0, s>>>(a, tiles, zero_rows_begin); break;
        case 2: k_rgcn_tile_fix<2><<<blocks, 256, 0, s>>>(a, tiles, zero_rows_begin); break;
        case 3: k_rgcn_tile_fix<3><<<blocks, 256, 0, s>>>(a, tiles, zero_rows_begin); break;
        default: k_rgcn_tile_fix<4><<<blocks, 256, 0, s>>>(a, tiles, zero_rows_begin); break;
    }
    return check_launch("k_rgcn_tile_fix");
}

// dW_r = sum over the edges of type r of norm_e X[src_e]^T dA[dst_e] (a10), per task of the type-major view (a task
// never crosses a type): the task's rows X[src] and dA[dst] are staged in chunks of kDwChunk edges (cp.async), warp
// w walks the contiguous stretch w/8 of a chunk with lane (ib, jb) owning the 2 x 4 block (2ib.., 4jb..) of the
// partial in registers, and the 8 warp partials are summed in warp order into part[t] (fixed order, no atomics).
// Replaces k_rgcn_dw_g for F_in, F_out <= 16, whose per-lane edge walk was latency-bound (r1/r2 AM launch lists).
namespace {
constexpr int kDwChunk = 512;
}

template <int FI4, int FO4>
__global__ void __launch_bounds__(256) k_rgcn_dw_tile(const RgcnDwTileArgs a) {
    constexpr int CH = kDwChunk, NW = 8;
    extern __shared__ float4 smem[];
    float4* xs = smem;                                       // [CH][FI4]
    float4* ds = xs + CH * FI4;                              // [CH][FO4]
    float* sw = reinterpret_cast<float*>(ds + CH * FO4);     // [CH]
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int ib = lane >> 2, jb = lane & 3;
    const int64_t t = blockIdx.x;
    const int es = __ldg(a.run_off + __ldg(a.task_run + t)), ee = __ldg(a.run_off + __ldg(a.task_run + t + 1));
    const bool own = 2 * ib < a.Fin && 4 * jb < a.Fout;
    float acc[2][4] = {{0.f, 0.f, 0.f, 0.f}, {0.f, 0.f, 0.f, 0.f}};
    for (int c0 = es; c0 < ee; c0 += CH) {
        const int nc = min(CH, ee - c0);
        for (int i = tid; i < nc; i += 256) {
            const int k = c0 + i;
            const int u = __ldg(a.src + k), d = __ldg(a.dst + k);
            sw[i] = a.norm_user ? __ldg(a.norm_user + __ldg(a.eid + k)) : __ldg(a.norm + k);
#pragma unroll
            for (int q = 0; q < FI4; ++q) cp_async16(xs + i * FI4 + q, a.X + (int64_t)u * a.ldx + 4 * q);
#pragma unroll
            for (int q = 0; q < FO4; ++q) cp_async16(ds + i * FO4 + q, a.dA + (int64_t)d * a.ldd + 4 * q);
        }
        cp_async_wait_all();
        __syncthreads();
        if (own) {
            const int p0 = nc * warp / NW, p1 = nc * (warp + 1) / NW;
            for (int p = p0; p < p1; ++p) {
                const float2 xv = *reinterpret_cast<const float2*>(reinterpret_cast<const float*>(xs + p * FI4) + 2 * ib);
                const float4 dv = ds[p * FO4 + (jb < FO4 ? jb : 0)];
                const float wg = sw[p];
                // the row padding is never read into a result
                const float x0 = xv.x * wg, x1 = 2 * ib + 1 < a.Fin ? xv.y * wg : 0.f;
                const float d[4] = {dv.x, 4 * jb + 1 < a.Fout ? dv.y : 0.f, 4 * jb + 2 < a.Fout ? dv.z : 0.f,
                                    4 * jb + 3 < a.Fout ? dv.w : 0.f};
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    acc[0][q] = fmaf(x0, d[q], acc[0][q]);
                    acc[1][q] = fmaf(x1, d[q], acc[1][q]);
                }
            }
        }
        __syncthreads();                                     // the chunk's slots are refilled next
    }
    const int FF = a.Fin * a.Fout;
    float* red = reinterpret_cast<float*>(smem);             // [NW][FF] (FF <= 256 floats: fits in xs)
    if (own)
#pragma unroll
        for (int i = 0; i < 2; ++i)
#pragma unroll
            for (int q = 0; q < 4; ++q)
                if (2 * ib + i < a.Fin && 4 * jb + q < a.Fout)
                    red[warp * FF + (2 * ib + i) * a.Fout + 4 * jb + q] = acc[i][q];
    __syncthreads();
    for (int e = tid; e < FF; e += 256) {
        float x = red[e];
#pragma unroll
        for (int w2 = 1; w2 < NW; ++w2) x += red[w2 * FF + e];
        a.part[t * FF + e] = x;
    }
}

seastar_status rgcn_dw_tile_launch(const RgcnDwTileArgs& a, cudaStream_t s) {
    if (a.n_tasks <= 0) return SEASTAR_OK;
    const int fi4 = (a.Fin + 3) / 4, fo4 = (a.Fout + 3) / 4;
    const size_t smem = (size_t)kDwChunk * ((fi4 + fo4) * 16 + 4);
    auto go = [&](auto kern) -> seastar_status {
        SS_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        launch_k(kern, dim3((unsigned)a.n_tasks), dim3(256), smem, s, a);
        return check_launch("k_rgcn_dw_tile");
    };
#define RGCN_DWT_FO(I4)                                      \
    switch (fo4) {                                           \
        case 1: return go(k_rgcn_dw_tile<I4, 1>);            \
        case 2: return go(k_rgcn_dw_tile<I4, 2>);            \
        case 3: return go(k_rgcn_dw_tile<I4, 3>);            \
        default: return go(k_rgcn_dw_tile<I4, 4>);           \
    }
    switch (fi4) {
        case 1: RGCN_DWT_FO(1)
        case 2: RGCN_DWT_FO(2)
        case 3: RGCN_DWT_FO(3)
        default: RGCN_DWT_FO(4)
    }
#undef RGCN_DWT_FO
}

}  // namespace seastar
