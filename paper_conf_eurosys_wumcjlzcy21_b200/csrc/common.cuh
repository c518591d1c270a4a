// common.cuh -- shared internals of libseastar.so (sm_100a).  Not part of the ABI.
#pragma once
#include <cmath>
#include <cstdlib>

#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <string>

#include "seastar.h"

namespace seastar {

// ----------------------------------------------------------------------------------------------
// error plumbing: thread-local message + status codes, no exceptions across the ABI
// ----------------------------------------------------------------------------------------------
void set_error(const char* fmt, ...);
seastar_status cuda_status(cudaError_t err, const char* where);
seastar_status check_launch(const char* where);
seastar_status check_device();   // sm_100 or UNSUPPORTED (cached per device)

#define SS_ARG(cond, ...)                                   \
    do {                                                    \
        if (!(cond)) {                                      \
            ::seastar::set_error(__VA_ARGS__);              \
            return SEASTAR_ERR_INVALID_ARGUMENT;            \
        }                                                   \
    } while (0)

#define SS_CUDA(call)                                                     \
    do {                                                                  \
        cudaError_t _e = (call);                                          \
        if (_e != cudaSuccess) return ::seastar::cuda_status(_e, #call);  \
    } while (0)

#define SS_TRY(expr)                          \
    do {                                      \
        seastar_status _s = (expr);           \
        if (_s != SEASTAR_OK) return _s;      \
    } while (0)

inline cudaStream_t to_stream(seastar_stream s) { return reinterpret_cast<cudaStream_t>(s); }

// ----------------------------------------------------------------------------------------------
// the graph handle (all index arrays are int32 on the device; E < 2^31 is validated at create)
// ----------------------------------------------------------------------------------------------
constexpr int kPow2Lo = 2, kPow2Classes = 15;   // degree thresholds 4 .. 65536 (long-row split, medium-row class)

struct IndexSet {
    int32_t* perm = nullptr;   // row -> vertex id            [n_rows]   (nullptr for LSF: identity)
    int32_t* off = nullptr;    // row offsets                 [n_rows+1]
    int32_t* nbr = nullptr;    // FWD: src id, REV: dst id     [n_edges]
    int32_t* eid = nullptr;    // user edge id                 [n_edges]
    int32_t* pos = nullptr;    // REV only: position in FWD (or LSF)
    int32_t* type = nullptr;   // edge type or nullptr
    float* norm = nullptr;     // R-GCN 1/c_{v,r} or nullptr
    int64_t n_rows = 0;
    int64_t n_edges = 0;
    int64_t bucket_rows[SEASTAR_NUM_BUCKETS] = {0, 0, 0, 0};
    int64_t max_deg = 0;
    int64_t pow2_rows[kPow2Classes] = {};   // rows with degree >= 2^(kPow2Lo + k) (rows are degree-sorted)
    int32_t* tile_row = nullptr;   // typed graphs: [2 n_tiles] first / last row of each kRgcnTileEdges-edge tile
};

// Type-major view of the FWD edges for the R-GCN weight gradient: edges sorted by (type, dst row,
// eid) and cut into (type, dst) runs; runs are grouped into tasks that never cross a type, so one
// warp can own dW_r partials in registers (deterministic, no atomics).
struct TypeMajor {
    int32_t* src = nullptr;       // [Ef] source id per edge
    int32_t* eid = nullptr;       // [Ef]
    float* norm = nullptr;        // [Ef] or nullptr
    int32_t* run_off = nullptr;   // [n_runs+1]
    int32_t* run_dst = nullptr;   // [n_runs] destination vertex id
    int32_t* task_run = nullptr;  // [n_tasks+1]
    int32_t* task_type = nullptr; // [n_tasks]
    int32_t* type_task = nullptr; // [R+1]
    int32_t* dst = nullptr;       // [Ef] destination vertex id of each edge (run boundaries = changes of dst in a task)
    int64_t n_runs = 0, n_tasks = 0;
};
// NEXT-1: an index set's rows with their edges re-ordered so that the edges whose neighbour is an
// owned vertex come first (stable, eid order inside each part).  The partitioned aggregation runs the owned-neighbour
// part from the rank's own table while the all-gather of the other ranks' rows is in flight, then the rest.
struct LocalSplit {
    int32_t* nbr = nullptr;    // [E] neighbour id, row-major like the index set (same off[])
    int32_t* eid = nullptr;    // [E] user edge id
    int32_t* lcnt = nullptr;   // [n_rows] owned-neighbour edges at the front of each row
};

constexpr int kTaskEdges = 512;   // edges per dW task (a task may exceed it only inside one run)

// Two-phase R-GCN (a7 forward on FWD, a10 dX on REV; rgcn.cu): an index set's edges in type-major order
// (type, row, eid) with, per edge, its type and its position in the index set's row order.  Phase 1 walks the edges
// in this order -- a warp's 32 consecutive edges share their type, so W_r reads from shared memory are broadcasts --
// and writes each edge's product norm_e * table[nbr_e] W_r to the edge's row-order position; phase 2 sums each
// row's contiguous products.
struct EdgeMajor {
    const int32_t* nbr = nullptr;   // [E] neighbour id (FWD: tm.src; REV: owned array)
    const int32_t* eid = nullptr;   // [E] user edge id
    const float* norm = nullptr;    // [E] 1/c_{v,r} or nullptr
    int32_t* type = nullptr;        // [E]
    int32_t* pos = nullptr;         // [E] position of the edge in the index set's row order (FWD / REV off[])
    int64_t n = 0;
};

}  // namespace seastar

struct seastar_graph_s {
    int device = 0;
    int64_t N = 0, E = 0, row_begin = 0, row_end = 0;
    int32_t R = 1;
    uint32_t flags = 0;
    bool partitioned = false;
    seastar::IndexSet fwd, rev, lsf;
    seastar::LocalSplit fsplit, rsplit;  // partitioned only: rows' edges with owned neighbours first (NEXT-1)
    seastar::TypeMajor tm;
    seastar::EdgeMajor fem, rem;     // two-phase R-GCN: FWD (forward) and REV (dX) edges in type-major order
    int32_t* rtm_nbr = nullptr;      // REV edges in type-major order (rem's edge arrays)
    int32_t* rtm_eid = nullptr;
    float* rtm_norm = nullptr;
    int32_t* indeg_loc = nullptr;    // [n_loc]
    int32_t* outdeg_loc = nullptr;   // [n_loc]
    void* pool = nullptr;            // single device allocation backing every array above
    size_t pool_bytes = 0;
    int64_t n_loc() const { return row_end - row_begin; }
};

namespace seastar {

constexpr int kBucketThreshold[SEASTAR_NUM_BUCKETS] = {1024, 32, 1, 0};

// ----------------------------------------------------------------------------------------------
// device helpers
// ----------------------------------------------------------------------------------------------
template <int VEC>
struct Vec;
template <>
struct Vec<4> {
    using T = float4;
};
template <>
struct Vec<1> {
    using T = float;
};

// read-only 128-bit / 32-bit loads through the non-coherent path
__device__ __forceinline__ float4 ldg4(const float* p) { return __ldg(reinterpret_cast<const float4*>(p)); }
__device__ __forceinline__ float ldg1(const float* p) { return __ldg(p); }

template <int VEC>
__device__ __forceinline__ void load_vec(const float* p, float (&v)[VEC]) {
    if constexpr (VEC == 4) {
        float4 t = ldg4(p);
        v[0] = t.x; v[1] = t.y; v[2] = t.z; v[3] = t.w;
    } else {
        v[0] = ldg1(p);
    }
}
template <int VEC>
__device__ __forceinline__ void store_vec(float* p, const float (&v)[VEC]) {
    if constexpr (VEC == 4) {
        *reinterpret_cast<float4*>(p) = make_float4(v[0], v[1], v[2], v[3]);
    } else {
        p[0] = v[0];
    }
}

// activation and its derivative expressed through the activation's output y
__device__ __forceinline__ float act_apply(int act, float x) {
    switch (act) {
        case SEASTAR_ACT_RELU: return x > 0.f ? x : 0.f;
        case SEASTAR_ACT_ELU: return x > 0.f ? x : expm1f(x);
        case SEASTAR_ACT_SIGMOID: return 1.f / (1.f + expf(-x));
        default: return x;
    }
}
__device__ __forceinline__ float act_grad_from_y(int act, float y) {
    switch (act) {
        case SEASTAR_ACT_RELU: return y > 0.f ? 1.f : 0.f;
        case SEASTAR_ACT_ELU: return y > 0.f ? 1.f : y + 1.f;
        case SEASTAR_ACT_SIGMOID: return y * (1.f - y);
        default: return 1.f;
    }
}

__host__ __device__ inline bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

// NEXT-3 dropout generator (reading #27): splitmix64's output function; a mask element keeps
// iff (sm64(key ^ i) >> 40) >= thr with key = sm64(seed ^ sm64((site << 32) | step))
__device__ __forceinline__ uint64_t sm64(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}
__device__ __forceinline__ uint64_t drop_key(uint64_t seed, uint32_t site, const int32_t* step) {
    const uint32_t st = step ? (uint32_t)__ldg(step) : 0u;
    return sm64(seed ^ sm64(((uint64_t)site << 32) | st));
}
__device__ __forceinline__ float drop_mult(uint64_t key, uint64_t i, uint32_t thr, float scale) {
    return (sm64(key ^ i) >> 40) >= thr ? scale : 0.f;
}
inline uint32_t drop_threshold(float p) { return (uint32_t)llround((double)p * 16777216.0); }
inline float drop_scale(float p) { return (float)(1.0 / (1.0 - (double)p)); }
// dropout fields (deid, dseed, dstep, dsite, dthr, dscale) of a kernel argument block from the ABI spec
// (NULL or p == 0: off, deid = nullptr); eid = the index set's user edge ids (the mask's counter)
template <typename Args>
inline void set_drop(Args& a, const seastar_dropout_spec* d, const int32_t* eid) {
    if (!d || d->p <= 0.f) { a.deid = nullptr; return; }
    a.deid = eid; a.dseed = d->seed; a.dstep = d->step; a.dsite = d->site;
    a.dthr = drop_threshold(d->p); a.dscale = drop_scale(d->p);
}

// ----------------------------------------------------------------------------------------------
// L2 residency of the gathered table.  Every edge of a graph kernel gathers a row of one table
// (T, dP, the GAT record D, X ...) that is 15-90 MB and therefore *could* live in the 126 MB L2, while
// the edge-index stream (4-8 B per edge, 0.5-1 GB) and the outputs stream through once.  Graph kernels read
// their index streams with evict-first loads (__ldcs).  The GAT backward and R-GCN launches can also carry an
// access-policy window over the gathered table (hits persist, misses stream) -- opt-in (SEASTAR_L2_PERSIST=1,
// l2_persist_bytes()): the persisting set-aside is device-wide and shrinks the L2 of every other kernel.
// ----------------------------------------------------------------------------------------------
struct L2Window {
    const void* base = nullptr;
    size_t bytes = 0;
};
extern thread_local L2Window t_l2win;

struct ScopedL2Window {
    L2Window saved;
    ScopedL2Window(const void* base, size_t bytes) : saved(t_l2win) { t_l2win = {base, bytes}; }
    ~ScopedL2Window() { t_l2win = saved; }
};

size_t l2_persist_bytes();
// out[(i / nc) * ldo + i % nc] = sum_b part[b * stride + i] for i < n: deterministic fp64 reduction of
// split partials (fixed order: 8 (or, for few outputs and many splits, 32) warp-strided lanes of splits, then
// the lanes in order); one block of
// 256 threads per 32 consecutive outputs, so the split count does not serialise the reduction
void reduce_splits(const float* part, int64_t nsplit, int64_t stride, int64_t n, int64_t nc, int64_t ldo, float* out,
                   cudaStream_t s);   // device set-aside for persisting lines (configured on first use), 0 if none

// out[s * width + e] = sum_{t in [seg_off[s], seg_off[s+1])} part[t * width + e] for s < nseg, e < width:
// deterministic fp64 segmented column sums (fixed task-to-thread assignment and merge order), one
// block per (segment, 32 columns).  Used for the per-type reduction of R-GCN task partials.
void seg_reduce_cols(const float* part, const int32_t* seg_off, int nseg, int width, float* out, cudaStream_t s);

template <typename... KArgs, typename... Args>
inline void launch_k(void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s, Args... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    cfg.attrs = attr;
    cfg.numAttrs = 0;
    const size_t persist = t_l2win.base && t_l2win.bytes ? l2_persist_bytes() : 0;
    if (persist) {
        const size_t win = t_l2win.bytes < ((size_t)128 << 20) ? t_l2win.bytes : ((size_t)128 << 20);
        attr[0].id = cudaLaunchAttributeAccessPolicyWindow;
        attr[0].val.accessPolicyWindow.base_ptr = const_cast<void*>(t_l2win.base);
        attr[0].val.accessPolicyWindow.num_bytes = win;
        attr[0].val.accessPolicyWindow.hitRatio = persist >= win ? 1.0f : (float)persist / (float)win;
        attr[0].val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        attr[0].val.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
        cfg.numAttrs = 1;
    }
    cudaLaunchKernelEx(&cfg, kernel, args...);
}

inline int num_sms() {
    static int sms = 0;
    if (!sms) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        if (sms <= 0) sms = 148;
    }
    return sms;
}

// "Long" rows of a row launch get a CTA of 8 warps in the same launch as the warp rows (PAPER.md L1253 CTA + Warp):
// every row whose edges exceed a quarter of one SM's share of the index set, which would keep one warp busy past
// the rest of the launch (CoraFull-shaped: ~250 edges).  Returns the number of leading (highest-degree) rows that
// qualify: degree >= the power of two at or above max(E / (4 #SMs), 128).  On the Reddit shape no row qualifies;
// giving its a3 hub class (degree >= 1024) CTAs was measured slower in the product kernels (r2 same-box A/B,
// profiles/r2/ab_long_rows.txt: GCN aggregation 0.68 -> 0.82 ms) although the NEXT-4 sweep's plain-sum kernel gains
// (profiles/r2/ablation.md).  SEASTAR_LONG_ROW=<degree> overrides the threshold (A/B runs; 0 disables).
inline int64_t long_rows(const IndexSet& x) {
    int64_t t = x.n_edges / (4 * (int64_t)num_sms());
    t = t > 128 ? t : 128;
    if (const char* env = getenv("SEASTAR_LONG_ROW")) {
        t = atoll(env);
        if (t <= 0) return 0;
    }
    int k = 0;
    while (k < kPow2Classes && ((int64_t)1 << (kPow2Lo + k)) < t) ++k;
    return k < kPow2Classes ? x.pow2_rows[k] : 0;
}

inline int pow2_ceil(int x) {
    int p = 1;
    while (p < x) p <<= 1;
    return p;
}

}  // namespace seastar
