// graph.cu -- library plumbing (errors, device check) and the a1-a3 preprocessing kernels:
// degree count, stable degree sort (row permutation), stable CSR transpose with edge-id carry,
// per-row type order, R-GCN normaliser and degree buckets (§6.1, Fig. 7,
// §6.3.3, §6.3.4, §6.3.5).
//
// Stability never comes from atomic order: every permutation is produced by CUB's LSD radix sort
// (stable by construction, ranks from prefix scans), so the result is bit-exact and unique.
#include <cub/cub.cuh>
#include <stdarg.h>
#include <stdlib.h>

#include <mutex>
#include <vector>

#include "common.cuh"
#include "rgcn_tile.cuh"

namespace seastar {

static thread_local std::string g_err;

void set_error(const char* fmt, ...) {
    char buf[1024];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof(buf), fmt, ap);
    va_end(ap);
    g_err = buf;
}

seastar_status cuda_status(cudaError_t err, const char* where) {
    set_error("%s: %s (%s)", where, cudaGetErrorString(err), cudaGetErrorName(err));
    return err == cudaErrorMemoryAllocation ? SEASTAR_ERR_OUT_OF_MEMORY : SEASTAR_ERR_CUDA;
}

seastar_status check_launch(const char* where) {
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_status(e, where);
    return SEASTAR_OK;
}

thread_local L2Window t_l2win;

size_t l2_persist_bytes() {
    static std::mutex mu;
    static long long per_dev[64];
    static bool init[64] = {false};
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return 0;
    std::lock_guard<std::mutex> lk(mu);
    if (!init[dev]) {
        init[dev] = true;
        per_dev[dev] = 0;
        int maxp = 0;
        // opt-in (SEASTAR_L2_PERSIST=1): the set-aside is device-wide and not stream-ordered, so once reserved it
        // shrinks the normal L2 for every later kernel -- measured on Reddit (r2): 13.92 ms/step with the window on
        // the GAT backward's records, 13.37 ms without it (stale persisting lines)
        const char* on = getenv("SEASTAR_L2_PERSIST");
        if (on != nullptr && on[0] == '1' &&
            cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, dev) == cudaSuccess && maxp > 0 &&
            cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, (size_t)maxp) == cudaSuccess)
            per_dev[dev] = maxp;
        cudaGetLastError();
    }
    return (size_t)per_dev[dev];
}

seastar_status check_device() {
    static std::mutex mu;
    static int ok_dev[64] = {0};   // 0 unknown, 1 ok, 2 unsupported
    int dev = 0;
    SS_CUDA(cudaGetDevice(&dev));
    if (dev < 0 || dev >= 64) return SEASTAR_ERR_UNSUPPORTED;
    std::lock_guard<std::mutex> lk(mu);
    if (ok_dev[dev] == 0) {
        int major = 0, minor = 0;
        SS_CUDA(cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev));
        SS_CUDA(cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev));
        ok_dev[dev] = (major == 10 && minor == 0) ? 1 : 2;
        if (ok_dev[dev] == 2) set_error("device %d is sm_%d%d; libseastar is built for sm_100a only", dev, major, minor);
    }
    return ok_dev[dev] == 1 ? SEASTAR_OK : SEASTAR_ERR_UNSUPPORTED;
}

// ----------------------------------------------------------------------------------------------
// kernels
// ----------------------------------------------------------------------------------------------
__global__ void k_validate(int64_t N, int64_t E, const int64_t* __restrict__ indptr,
                           const int64_t* __restrict__ indices, const int32_t* __restrict__ etypes, int32_t R,
                           int* __restrict__ flag) {
    int64_t n = N + 1 > E ? N + 1 : E;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        int bad = 0;
        if (i == 0 && (indptr[0] != 0 || indptr[N] != E)) bad |= 1;
        if (i < N && indptr[i] > indptr[i + 1]) bad |= 2;
        if (i < E) {
            int64_t s = indices[i];
            if (s < 0 || s >= N) bad |= 4;
            if (etypes && (etypes[i] < 0 || etypes[i] >= R)) bad |= 8;
        }
        if (bad) atomicOr(flag, bad);
    }
}

// warp per vertex: dst[e] = v for e in [indptr[v], indptr[v+1])
__global__ void k_fill_dst(int64_t N, const int64_t* __restrict__ indptr, int32_t* __restrict__ dst) {
    int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    int lane = threadIdx.x & 31;
    for (int64_t v = warp; v < N; v += ((int64_t)gridDim.x * blockDim.x) >> 5)
        for (int64_t e = indptr[v] + lane; e < indptr[v + 1]; e += 32) dst[e] = (int32_t)v;
}

// out-degree histogram (integer atomics: the counts do not depend on the order) and the number
// of edges whose source lies in [rb, re)
__global__ void k_outdeg(int64_t E, const int64_t* __restrict__ indices, int32_t* __restrict__ outdeg, int64_t rb,
                         int64_t re, unsigned long long* __restrict__ n_owned_src) {
    unsigned long long local = 0;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < E; e += (int64_t)gridDim.x * blockDim.x) {
        int64_t s = indices[e];
        atomicAdd(&outdeg[s], 1);
        local += (s >= rb && s < re);
    }
    for (int o = 16; o; o >>= 1) local += __shfl_xor_sync(0xffffffffu, local, o);
    if ((threadIdx.x & 31) == 0 && local) atomicAdd(n_owned_src, local);
}

// sort keys for the owned vertices: ~deg sorts ascending == degree descending; value = vertex id
__global__ void k_vertex_keys(int64_t n_loc, int64_t rb, const int64_t* __restrict__ indptr,
                              const int32_t* __restrict__ outdeg, uint32_t* __restrict__ keys,
                              int32_t* __restrict__ vals, int32_t* __restrict__ deg_loc) {
    int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i >= n_loc) return;
    int64_t v = rb + i;
    uint32_t d = indptr ? (uint32_t)(indptr[v + 1] - indptr[v]) : (uint32_t)outdeg[v];
    keys[i] = ~d;
    vals[i] = (int32_t)v;
    if (deg_loc) deg_loc[i] = (int32_t)d;
}

// rowdeg[k] = deg(perm[k]) for k < n, rowdeg[n] = 0 (so an exclusive scan gives n+1 offsets)
__global__ void k_row_deg(int64_t n, int64_t rb, const int32_t* __restrict__ perm, const int32_t* __restrict__ deg_loc,
                          int32_t* __restrict__ rowdeg) {
    int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (k < n) rowdeg[k] = deg_loc[perm[k] - rb];
    if (k == n) rowdeg[n] = 0;
}

// row ranks: inv[perm[k] - rb] = k
__global__ void k_invert(int64_t n, int64_t rb, const int32_t* __restrict__ perm, int32_t* __restrict__ inv) {
    int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (k < n) inv[perm[k] - rb] = (int32_t)k;
}

// warp per forward row: copy the user's in-edges of perm[k] (already in eid order)
__global__ void k_fill_fwd(int64_t n, const int32_t* __restrict__ perm, const int32_t* __restrict__ off,
                           const int64_t* __restrict__ indptr, const int64_t* __restrict__ indices,
                           const int32_t* __restrict__ etypes, int32_t* __restrict__ src, int32_t* __restrict__ eid,
                           int32_t* __restrict__ typ, uint64_t* __restrict__ key64, int tbits) {
    int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    int lane = threadIdx.x & 31;
    for (int64_t k = warp; k < n; k += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        int64_t v = perm[k];
        int64_t b = indptr[v], d = indptr[v + 1] - b, o = off[k];
        for (int64_t j = lane; j < d; j += 32) {
            int64_t e = b + j;
            src[o + j] = (int32_t)indices[e];
            eid[o + j] = (int32_t)e;
            if (typ) typ[o + j] = etypes[e];
            if (key64) key64[o + j] = ((uint64_t)k << tbits) | (uint64_t)etypes[e];
        }
    }
}

__global__ void k_iota(int64_t n, int32_t* __restrict__ out) {
    int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i < n) out[i] = (int32_t)i;
}

// dst[i] = src[idx[i]] for int32 arrays
__global__ void k_gather_i32(int64_t n, const int32_t* __restrict__ idx, const int32_t* __restrict__ src,
                             int32_t* __restrict__ dst) {
    int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i < n) dst[i] = src[idx[i]];
}
__global__ void k_gather_i32_from64(int64_t n, const int32_t* __restrict__ idx, const int64_t* __restrict__ src,
                                    int32_t* __restrict__ dst) {
    int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i < n) dst[i] = (int32_t)src[idx[i]];
}
__global__ void k_gather_f32(int64_t n, const int32_t* __restrict__ idx, const float* __restrict__ src,
                             float* __restrict__ dst) {
    int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i < n) dst[i] = src[idx[i]];
}
// scatter position map: pos_of[eid[j]] = j
__global__ void k_scatter_pos(int64_t n, const int32_t* __restrict__ eid, int32_t* __restrict__ pos_of) {
    int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (j < n) pos_of[eid[j]] = (int32_t)j;
}

// edge keys for the reverse sort: key = (rank of src) [<< tbits | type], over the given edge list
__global__ void k_rev_keys32(int64_t n, const int32_t* __restrict__ eids, const int64_t* __restrict__ indices,
                             const int32_t* __restrict__ inv_rev, int64_t rb, uint32_t* __restrict__ key) {
    int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i < n) key[i] = (uint32_t)inv_rev[indices[eids[i]] - rb];
}
__global__ void k_rev_keys64(int64_t n, const int32_t* __restrict__ eids, const int64_t* __restrict__ indices,
                             const int32_t* __restrict__ etypes, const int32_t* __restrict__ inv_rev, int64_t rb,
                             int tbits, uint64_t* __restrict__ key) {
    int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i < n) {
        int32_t e = eids[i];
        uint64_t t = etypes ? (uint64_t)etypes[e] : 0;
        key[i] = ((uint64_t)inv_rev[indices[e] - rb] << tbits) | t;
    }
}
// keys (dst [<< tbits | type]) over an edge list, for the LSF order and the R-GCN run lengths
__global__ void k_dst_keys64(int64_t n, const int32_t* __restrict__ eids, const int32_t* __restrict__ dst,
                             const int32_t* __restrict__ etypes, int tbits, uint64_t* __restrict__ key) {
    int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i < n) {
        int32_t e = eids ? eids[i] : (int32_t)i;
        uint64_t t = etypes ? (uint64_t)etypes[e] : 0;
        key[i] = ((uint64_t)dst[e] << tbits) | t;
    }
}
__global__ void k_owned_src_flags(int64_t E, const int64_t* __restrict__ indices, int64_t rb, int64_t re,
                                  uint8_t* __restrict__ flags) {
    int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (e < E) flags[e] = (indices[e] >= rb && indices[e] < re) ? 1 : 0;
}
__global__ void k_hist_dst(int64_t n, const int32_t* __restrict__ eids, const int32_t* __restrict__ dst,
                           int32_t* __restrict__ cnt) {
    int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i < n) atomicAdd(&cnt[dst[eids[i]]], 1);
}

// R-GCN normaliser: thread per vertex over its (type-sorted) segment of the user CSR; each run of
// equal type has length c_{v,r}; norm_by_eid[e] = 1 / c_{v,r}
__global__ void k_rgcn_runs(int64_t N, const int64_t* __restrict__ indptr, const int32_t* __restrict__ sorted_eid,
                            const int32_t* __restrict__ etypes, float* __restrict__ norm_by_eid) {
    int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (v >= N) return;
    int64_t b = indptr[v], e_end = indptr[v + 1];
    int64_t run = b;
    for (int64_t p = b; p < e_end; ++p) {
        bool last = (p + 1 == e_end) || (etypes[sorted_eid[p + 1]] != etypes[sorted_eid[p]]);
        if (last) {
            float w = 1.0f / (float)(p + 1 - run);
            for (int64_t q = run; q <= p; ++q) norm_by_eid[sorted_eid[q]] = w;
            run = p + 1;
        }
    }
}

// long-row classes over degree-sorted rows: out[k] = #rows with deg >= 2^(kPow2Lo + k)
__global__ void k_pow2_rows(int64_t n, const int32_t* __restrict__ off, long long* __restrict__ out) {
    int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (k >= n) return;
    const int32_t d = off[k + 1] - off[k];
    const int32_t dn = (k + 1 < n) ? off[k + 2] - off[k + 1] : -1;
    for (int i = 0; i < kPow2Classes; ++i) {
        const int32_t th = 1 << (kPow2Lo + i);
        if (d >= th && dn < th) out[i] = k + 1;
    }
}

// degree buckets over degree-sorted rows: out[i] = #rows with deg >= threshold[i]; out[4] = max degree
// R-GCN edge-balanced tiles (rgcn_tile.cu): tile_row[2t] / [2t+1] = the first / last row with an edge in tile t =
// [t * kRgcnTileEdges, min((t + 1) * kRgcnTileEdges, E)) (rows with edges come first: rows are degree-sorted)
__global__ void k_tile_rows(int64_t n, const int32_t* __restrict__ off, int32_t* __restrict__ tr) {
    const int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (r >= n) return;
    const int64_t b = off[r], e = off[r + 1], E = off[n];
    if (b == e) return;
    const int64_t tb = b / kRgcnTileEdges, te = (e - 1) / kRgcnTileEdges;
    if (b % kRgcnTileEdges == 0 || r == 0) tr[2 * tb] = (int32_t)r;        // first row of tile tb
    for (int64_t t = tb + 1; t <= te; ++t) tr[2 * t] = (int32_t)r;         // the row continues into tile t
    for (int64_t t = tb; t < te; ++t) tr[2 * t + 1] = (int32_t)r;          // ... and covers tile t's last edge
    const int64_t end_te = (te + 1) * kRgcnTileEdges < E ? (te + 1) * kRgcnTileEdges : E;
    if (e == end_te) tr[2 * te + 1] = (int32_t)r;
}

static seastar_status tile_rows(int64_t n, const int32_t* off, int32_t* tr, cudaStream_t s) {
    if (n > 0) k_tile_rows<<<(unsigned)((n + 255) / 256), 256, 0, s>>>(n, off, tr);
    return check_launch("k_tile_rows");
}

__global__ void k_buckets(int64_t n, const int32_t* __restrict__ off, long long* __restrict__ out) {
    int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (k >= n) return;
    int32_t d = off[k + 1] - off[k];
    int32_t dn = (k + 1 < n) ? off[k + 2] - off[k + 1] : -1;
    const int th[SEASTAR_NUM_BUCKETS] = {1024, 32, 1, 0};
    for (int i = 0; i < SEASTAR_NUM_BUCKETS; ++i)
        if (d >= th[i] && dn < th[i]) out[i] = k + 1;
    if (k == 0) out[SEASTAR_NUM_BUCKETS] = d;
}

__global__ void k_degree_norms(int64_t n, const int32_t* __restrict__ indeg, const int32_t* __restrict__ outdeg,
                               int mode, float* __restrict__ src_norm, float* __restrict__ dst_norm) {
    int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    int32_t di = indeg[i] > 1 ? indeg[i] : 1;
    int32_t dout = outdeg[i] > 1 ? outdeg[i] : 1;
    float ni = 1.0f / sqrtf((float)di);
    if (dst_norm) dst_norm[i] = ni;
    if (src_norm) src_norm[i] = mode == SEASTAR_NORM_IN ? ni : 1.0f / sqrtf((float)dout);
}

// ---- type-major view (R-GCN dW): edges by (type, fwd row, eid), cut into runs and tasks --------
__global__ void k_row_index(int64_t n, const int32_t* __restrict__ off, int32_t* __restrict__ rowidx) {
    const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    for (int64_t k = warp; k < n; k += ((int64_t)gridDim.x * blockDim.x) >> 5)
        for (int64_t p = off[k] + lane; p < off[k + 1]; p += 32) rowidx[p] = (int32_t)k;
}
__global__ void k_tm_keys(int64_t n, const int32_t* __restrict__ rowidx, const int32_t* __restrict__ typ, int rbits,
                          uint64_t* __restrict__ key) {
    const int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (p < n) key[p] = ((uint64_t)typ[p] << rbits) | (uint64_t)rowidx[p];
}
__global__ void k_tm_fill(int64_t n, const int32_t* __restrict__ pos, const int32_t* __restrict__ src,
                          const int32_t* __restrict__ eid, const float* __restrict__ norm, int32_t* __restrict__ tsrc,
                          int32_t* __restrict__ teid, float* __restrict__ tnorm, const int32_t* __restrict__ rowidx = nullptr,
                          const int32_t* __restrict__ perm = nullptr, int32_t* __restrict__ tdst = nullptr) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    const int32_t p = pos[i];
    tsrc[i] = src[p];
    teid[i] = eid[p];
    if (tnorm) tnorm[i] = norm[p];
    if (tdst) tdst[i] = perm[rowidx[p]];
}
__global__ void k_tm_run_heads(int64_t n, const uint64_t* __restrict__ key, int32_t* __restrict__ head) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i < n) head[i] = (i == 0 || key[i] != key[i - 1]) ? 1 : 0;
}
// runs: run r starts at the r-th head; meta[0] = #runs
__global__ void k_tm_runs(int64_t n, const uint64_t* __restrict__ key, const int32_t* __restrict__ head,
                          const int32_t* __restrict__ rid, int rbits, const int32_t* __restrict__ perm,
                          int32_t* __restrict__ run_off, int32_t* __restrict__ run_dst, int32_t* __restrict__ run_type,
                          long long* __restrict__ meta) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    if (head[i]) {
        const int32_t r = rid[i] - 1;
        const uint64_t k = key[i];
        run_off[r] = (int32_t)i;
        run_dst[r] = perm[k & ((1ull << rbits) - 1)];
        run_type[r] = (int32_t)(k >> rbits);
    }
    if (i == n - 1) {
        run_off[rid[i]] = (int32_t)n;
        meta[0] = rid[i];
    }
}
// a task starts at run 0, at every type change, and whenever a run starts in a new kTaskEdges block
__global__ void k_tm_task_heads(int64_t bound, const long long* __restrict__ meta, const int32_t* __restrict__ run_off,
                                const int32_t* __restrict__ run_type, int ke, int32_t* __restrict__ thead) {
    const int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (r >= bound) return;
    const int64_t nr = meta[0];
    if (r >= nr) { thead[r] = 0; return; }
    thead[r] = (r == 0 || run_type[r] != run_type[r - 1] || run_off[r] / ke != run_off[r - 1] / ke) ? 1 : 0;
}
__global__ void k_tm_tasks(int64_t bound, long long* __restrict__ meta, const int32_t* __restrict__ thead,
                           const int32_t* __restrict__ tid, const int32_t* __restrict__ run_type,
                           int32_t* __restrict__ task_run, int32_t* __restrict__ task_type, int32_t* __restrict__ cnt) {
    const int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    const int64_t nr = meta[0];
    if (r >= bound || r >= nr) return;
    if (thead[r]) {
        const int32_t t = tid[r] - 1;
        task_run[t] = (int32_t)r;
        task_type[t] = run_type[r];
        atomicAdd(&cnt[run_type[r]], 1);   // integer count per type: order-independent
    }
    if (r == nr - 1) {
        task_run[tid[r]] = (int32_t)nr;
        meta[1] = tid[r];
    }
}

// ---- NEXT-1 local-first split: key = row << 1 | (neighbour not owned); owned-neighbour counts per row
__global__ void k_split_keys(int64_t n, const int32_t* __restrict__ rowidx, const int32_t* __restrict__ nbr,
                             int64_t rb, int64_t re, uint64_t* __restrict__ key, int32_t* __restrict__ lcnt) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    const int64_t u = nbr[i];
    const bool own = u >= rb && u < re;
    key[i] = ((uint64_t)rowidx[i] << 1) | (own ? 0u : 1u);
    if (own) atomicAdd(&lcnt[rowidx[i]], 1);   // integer count per row: order-independent
}

// ---- two-phase R-GCN edge-major views: the type of every type-major edge (from its sort key)
__global__ void k_em_type(int64_t n, const uint64_t* __restrict__ key, int rbits, int32_t* __restrict__ type) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i < n) type[i] = (int32_t)(key[i] >> rbits);
}

// ----------------------------------------------------------------------------------------------
// host helpers
// ----------------------------------------------------------------------------------------------
static inline unsigned grid_for(int64_t n, int threads) { return (unsigned)((n + threads - 1) / threads); }
static inline int bit_width(uint64_t x) {
    int b = 0;
    while (x) { ++b; x >>= 1; }
    return b;
}

// tiny RAII set of stream-ordered temporaries
struct Temps {
    cudaStream_t s;
    std::vector<void*> ptrs;
    explicit Temps(cudaStream_t st) : s(st) {}
    ~Temps() {
        for (void* p : ptrs) cudaFreeAsync(p, s);
    }
    template <typename T>
    cudaError_t alloc(T** p, size_t count) {
        void* raw = nullptr;
        cudaError_t e = cudaMallocAsync(&raw, count * sizeof(T) + 16, s);
        if (e == cudaSuccess) ptrs.push_back(raw);
        *p = reinterpret_cast<T*>(raw);
        return e;
    }
};

template <typename K>
static seastar_status radix_sort_pairs(Temps& t, const K* kin, K* kout, const int32_t* vin, int32_t* vout,
                                       int64_t n, int end_bit) {
    if (n == 0) return SEASTAR_OK;
    size_t bytes = 0;
    SS_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, bytes, kin, kout, vin, vout, (int)n, 0, end_bit, t.s));
    void* tmp = nullptr;
    SS_CUDA(t.alloc(reinterpret_cast<char**>(&tmp), bytes));
    SS_CUDA(cub::DeviceRadixSort::SortPairs(tmp, bytes, kin, kout, vin, vout, (int)n, 0, end_bit, t.s));
    return SEASTAR_OK;
}

static seastar_status exclusive_sum(Temps& t, const int32_t* in, int32_t* out, int64_t n) {
    size_t bytes = 0;
    SS_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, bytes, in, out, (int)n, t.s));
    void* tmp = nullptr;
    SS_CUDA(t.alloc(reinterpret_cast<char**>(&tmp), bytes));
    SS_CUDA(cub::DeviceScan::ExclusiveSum(tmp, bytes, in, out, (int)n, t.s));
    return SEASTAR_OK;
}

static seastar_status inclusive_sum(Temps& t, const int32_t* in, int32_t* out, int64_t n) {
    size_t bytes = 0;
    SS_CUDA(cub::DeviceScan::InclusiveSum(nullptr, bytes, in, out, (int)n, t.s));
    void* tmp = nullptr;
    SS_CUDA(t.alloc(reinterpret_cast<char**>(&tmp), bytes));
    SS_CUDA(cub::DeviceScan::InclusiveSum(tmp, bytes, in, out, (int)n, t.s));
    return SEASTAR_OK;
}

// sort owned vertices by (degree desc, id asc) and build the row offsets
static seastar_status sort_rows(Temps& t, int64_t n_loc, int64_t rb, const int64_t* indptr, const int32_t* outdeg,
                                int32_t* deg_loc, int32_t* perm, int32_t* off) {
    cudaStream_t s = t.s;
    uint32_t *kin, *kout;
    int32_t *vin, *rowdeg;
    SS_CUDA(t.alloc(&kin, n_loc + 1));
    SS_CUDA(t.alloc(&kout, n_loc + 1));
    SS_CUDA(t.alloc(&vin, n_loc + 1));
    SS_CUDA(t.alloc(&rowdeg, n_loc + 1));
    if (n_loc > 0) {
        k_vertex_keys<<<grid_for(n_loc, 256), 256, 0, s>>>(n_loc, rb, indptr, outdeg, kin, vin, deg_loc);
        SS_TRY(check_launch("k_vertex_keys"));
        SS_TRY(radix_sort_pairs<uint32_t>(t, kin, kout, vin, perm, n_loc, 32));
    }
    k_row_deg<<<grid_for(n_loc + 1, 256), 256, 0, s>>>(n_loc, rb, perm, deg_loc, rowdeg);
    SS_TRY(check_launch("k_row_deg"));
    SS_TRY(exclusive_sum(t, rowdeg, off, n_loc + 1));
    return SEASTAR_OK;
}

}  // namespace seastar

using namespace seastar;

#define CK(expr)                                                            \
    do {                                                                    \
        cudaError_t _e = (expr);                                            \
        if (_e != cudaSuccess) return fail(cuda_status(_e, #expr));         \
    } while (0)
#define CKS(expr)                                                           \
    do {                                                                    \
        seastar_status _s = (expr);                                         \
        if (_s != SEASTAR_OK) return fail(_s);                              \
    } while (0)
#define CKS_LAUNCH(name) CKS(check_launch(name))

extern "C" {

const char* seastar_last_error(void) { return g_err.c_str(); }
int32_t seastar_abi_version(void) { return SEASTAR_ABI_VERSION; }
seastar_status seastar_device_check(void) { return check_device(); }

seastar_status seastar_graph_create(int64_t N, int64_t E, const int64_t* indptr, const int64_t* indices,
                                    const int32_t* etypes, int32_t num_etypes, int64_t row_begin, int64_t row_end,
                                    uint32_t flags, seastar_stream stream, seastar_graph* out) {
    SS_ARG(out != nullptr, "graph_create: out is NULL");
    *out = nullptr;
    SS_ARG(N >= 0 && N < (1LL << 31) - 1, "graph_create: N=%lld out of range [0, 2^31-1)", (long long)N);
    SS_ARG(E >= 0 && E < (1LL << 31) - 1, "graph_create: E=%lld out of range [0, 2^31-1)", (long long)E);
    SS_ARG(indptr != nullptr, "graph_create: indptr is NULL");
    SS_ARG(E == 0 || indices != nullptr, "graph_create: indices is NULL");
    SS_ARG(0 <= row_begin && row_begin <= row_end && row_end <= N, "graph_create: bad row range [%lld,%lld)",
           (long long)row_begin, (long long)row_end);
    SS_ARG(etypes == nullptr || (num_etypes >= 1 && num_etypes <= (1 << 20)),
           "graph_create: num_etypes=%d out of range [1, 2^20]", num_etypes);
    SS_ARG((flags & ~SEASTAR_GRAPH_RGCN_NORM) == 0, "graph_create: unknown flags 0x%x", flags);
    SS_TRY(check_device());

    cudaStream_t s = to_stream(stream);
    const int32_t R = etypes ? num_etypes : 1;
    const int tbits = etypes ? bit_width((uint64_t)(R - 1)) : 0;
    const int64_t n_loc = row_end - row_begin;
    const bool part = !(row_begin == 0 && row_end == N);
    const bool want_norm = (flags & SEASTAR_GRAPH_RGCN_NORM) != 0;

    seastar_graph g = new (std::nothrow) seastar_graph_s();
    if (!g) { set_error("graph_create: host allocation failed"); return SEASTAR_ERR_OUT_OF_MEMORY; }
    auto fail = [&](seastar_status st) {
        if (g->pool) cudaFree(g->pool);
        delete g;
        return st;
    };
    cudaGetDevice(&g->device);
    g->N = N; g->E = E; g->row_begin = row_begin; g->row_end = row_end; g->R = R; g->flags = flags;
    g->partitioned = part;

    {
        Temps t(s);
        // ---- validation + out-degrees ------------------------------------------------------------
        int* d_flag;
        unsigned long long* d_nown;
        int32_t* outdeg;
        int64_t* d_ip2;
        CK(t.alloc(&d_flag, 1));
        CK(t.alloc(&d_nown, 1));
        CK(t.alloc(&outdeg, N + 1));
        CK(t.alloc(&d_ip2, 2));
        CK(cudaMemsetAsync(d_flag, 0, sizeof(int), s));
        CK(cudaMemsetAsync(d_nown, 0, sizeof(unsigned long long), s));
        CK(cudaMemsetAsync(outdeg, 0, sizeof(int32_t) * (N + 1), s));
        k_validate<<<4 * num_sms(), 256, 0, s>>>(N, E, indptr, indices, etypes, R, d_flag);
        CKS(check_launch("k_validate"));
        int h_flag = 0;
        CK(cudaMemcpyAsync(&h_flag, d_flag, sizeof(int), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        if (h_flag) {
            set_error("graph_create: invalid graph (%s%s%s%s)", (h_flag & 1) ? "indptr[0]!=0 or indptr[N]!=E; " : "",
                      (h_flag & 2) ? "indptr not monotone; " : "", (h_flag & 4) ? "indices out of [0,N); " : "",
                      (h_flag & 8) ? "etypes out of [0,R); " : "");
            return fail(SEASTAR_ERR_INVALID_GRAPH);
        }
        if (E > 0) {
            k_outdeg<<<4 * num_sms(), 256, 0, s>>>(E, indices, outdeg, row_begin, row_end, d_nown);
            CKS(check_launch("k_outdeg"));
        }
        unsigned long long h_nown = 0;
        int64_t ip2[2] = {0, 0};
        CK(cudaMemcpyAsync(&h_nown, d_nown, sizeof(h_nown), cudaMemcpyDeviceToHost, s));
        CK(cudaMemcpyAsync(&ip2[0], indptr + row_begin, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
        CK(cudaMemcpyAsync(&ip2[1], indptr + row_end, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        const int64_t Ef = ip2[1] - ip2[0];
        const int64_t Er = (int64_t)h_nown;

        // ---- persistent pool ---------------------------------------------------------------------
        struct Slot { void** p; size_t bytes; };
        std::vector<Slot> slots;
        auto want = [&](auto** p, size_t count, bool on) {
            if (on) slots.push_back({reinterpret_cast<void**>(p), count * sizeof(**p)});
        };
        want(&g->fwd.perm, n_loc, true);
        want(&g->fwd.off, n_loc + 1, true);
        want(&g->fwd.nbr, Ef, true);
        want(&g->fwd.eid, Ef, true);
        want(&g->fwd.type, Ef, etypes != nullptr);
        want(&g->fwd.norm, Ef, want_norm);
        want(&g->rev.perm, n_loc, true);
        want(&g->rev.off, n_loc + 1, true);
        want(&g->rev.nbr, Er, true);
        want(&g->rev.eid, Er, true);
        want(&g->rev.pos, Er, true);
        want(&g->rev.type, Er, etypes != nullptr);
        want(&g->rev.norm, Er, want_norm);
        const int64_t fwd_tiles = (Ef + kRgcnTileEdges - 1) / kRgcnTileEdges;
        const int64_t rev_tiles = (Er + kRgcnTileEdges - 1) / kRgcnTileEdges;
        want(&g->fwd.tile_row, 2 * fwd_tiles + 2, etypes != nullptr);
        want(&g->rev.tile_row, 2 * rev_tiles + 2, etypes != nullptr);
        want(&g->lsf.off, N + 1, part);
        want(&g->lsf.eid, Er, part);
        want(&g->fsplit.nbr, Ef, part);
        want(&g->fsplit.eid, Ef, part);
        want(&g->fsplit.lcnt, n_loc, part);
        want(&g->rsplit.nbr, Er, part);
        want(&g->rsplit.eid, Er, part);
        want(&g->rsplit.lcnt, n_loc, part);
        want(&g->indeg_loc, n_loc, true);
        want(&g->outdeg_loc, n_loc, true);
        const bool tm_on = etypes != nullptr && Ef > 0;
        want(&g->tm.src, Ef, tm_on);
        want(&g->tm.eid, Ef, tm_on);
        want(&g->tm.norm, Ef, tm_on && want_norm);
        want(&g->tm.run_off, Ef + 1, tm_on);
        want(&g->tm.run_dst, Ef, tm_on);
        want(&g->tm.task_run, Ef + 1, tm_on);
        want(&g->tm.task_type, Ef, tm_on);
        want(&g->tm.type_task, R + 1, tm_on);
        want(&g->tm.dst, Ef, tm_on);
        const bool rtm_on = etypes != nullptr && Er > 0;
        want(&g->fem.type, Ef, tm_on);
        want(&g->fem.pos, Ef, tm_on);
        want(&g->rtm_nbr, Er, rtm_on);
        want(&g->rtm_eid, Er, rtm_on);
        want(&g->rtm_norm, Er, rtm_on && want_norm);
        want(&g->rem.type, Er, rtm_on);
        want(&g->rem.pos, Er, rtm_on);
        size_t total = 0;
        for (auto& sl : slots) total += (sl.bytes + 255) & ~size_t(255);
        {
            cudaError_t e = cudaMalloc(&g->pool, total ? total : 256);
            if (e != cudaSuccess) return fail(cuda_status(e, "cudaMalloc(graph pool)"));
        }
        g->pool_bytes = total;
        {
            char* base = static_cast<char*>(g->pool);
            for (auto& sl : slots) {
                *sl.p = base;
                base += (sl.bytes + 255) & ~size_t(255);
            }
        }
        g->fwd.n_rows = n_loc; g->fwd.n_edges = Ef;
        g->rev.n_rows = n_loc; g->rev.n_edges = Er;
        g->lsf.n_rows = part ? N : 0; g->lsf.n_edges = part ? Er : 0;

        // ---- shared temporaries -----------------------------------------------------------------
        int32_t* dst = nullptr;
        if (t.alloc(&dst, E + 1) != cudaSuccess) return fail(cuda_status(cudaErrorMemoryAllocation, "temps"));
        if (N > 0) {
            k_fill_dst<<<8 * num_sms(), 256, 0, s>>>(N, indptr, dst);
            CKS_LAUNCH("k_fill_dst");
        }

        // ---- a1: forward CSR ----------------------------------------------------------------------
        CKS(sort_rows(t, n_loc, row_begin, indptr, nullptr, g->indeg_loc, g->fwd.perm, g->fwd.off));
        if (g->fwd.tile_row) CKS(tile_rows(n_loc, g->fwd.off, g->fwd.tile_row, s));
        if (!etypes) {
            if (n_loc > 0) {
                k_fill_fwd<<<8 * num_sms(), 256, 0, s>>>(n_loc, g->fwd.perm, g->fwd.off, indptr, indices, nullptr,
                                                         g->fwd.nbr, g->fwd.eid, nullptr, nullptr, 0);
                CKS_LAUNCH("k_fill_fwd");
            }
        } else if (Ef > 0) {
            // fill in (row, eid) order, then a stable sort by (row, type) keeps eid order per type
            int32_t *src0, *eid0, *typ0, *iota, *order;
            uint64_t *k0, *k1;
            if (t.alloc(&src0, Ef) || t.alloc(&eid0, Ef) || t.alloc(&typ0, Ef) || t.alloc(&iota, Ef) ||
                t.alloc(&order, Ef) || t.alloc(&k0, Ef) || t.alloc(&k1, Ef))
                return fail(cuda_status(cudaErrorMemoryAllocation, "temps(fwd typed)"));
            k_fill_fwd<<<8 * num_sms(), 256, 0, s>>>(n_loc, g->fwd.perm, g->fwd.off, indptr, indices, etypes, src0, eid0,
                                                     typ0, k0, tbits);
            k_iota<<<grid_for(Ef, 256), 256, 0, s>>>(Ef, iota);
            CKS_LAUNCH("k_fill_fwd(typed)");
            CKS(radix_sort_pairs<uint64_t>(t, k0, k1, iota, order, Ef, tbits + bit_width((uint64_t)n_loc)));
            k_gather_i32<<<grid_for(Ef, 256), 256, 0, s>>>(Ef, order, src0, g->fwd.nbr);
            k_gather_i32<<<grid_for(Ef, 256), 256, 0, s>>>(Ef, order, eid0, g->fwd.eid);
            k_gather_i32<<<grid_for(Ef, 256), 256, 0, s>>>(Ef, order, typ0, g->fwd.type);
            CKS_LAUNCH("k_gather(fwd)");
        }

        // ---- a2: reverse CSR ----------------------------------------------------------------------
        CKS(sort_rows(t, n_loc, row_begin, nullptr, outdeg, g->outdeg_loc, g->rev.perm, g->rev.off));
        if (g->rev.tile_row) CKS(tile_rows(n_loc, g->rev.off, g->rev.tile_row, s));
        int32_t *inv_rev, *sel_eid;
        if (t.alloc(&inv_rev, n_loc + 1) || t.alloc(&sel_eid, Er + 1))
            return fail(cuda_status(cudaErrorMemoryAllocation, "temps(rev)"));
        if (n_loc > 0) k_invert<<<grid_for(n_loc, 256), 256, 0, s>>>(n_loc, row_begin, g->rev.perm, inv_rev);
        // edges with an owned source, in eid order
        if (!part) {
            if (E > 0) k_iota<<<grid_for(E, 256), 256, 0, s>>>(E, sel_eid);
        } else if (E > 0) {
            uint8_t* fl;
            int32_t *iota, *nsel;
            if (t.alloc(&fl, E) || t.alloc(&iota, E) || t.alloc(&nsel, 1))
                return fail(cuda_status(cudaErrorMemoryAllocation, "temps(select)"));
            k_owned_src_flags<<<grid_for(E, 256), 256, 0, s>>>(E, indices, row_begin, row_end, fl);
            k_iota<<<grid_for(E, 256), 256, 0, s>>>(E, iota);
            size_t bytes = 0;
            cub::DeviceSelect::Flagged(nullptr, bytes, iota, fl, sel_eid, nsel, (int)E, s);
            void* tmp;
            if (t.alloc(reinterpret_cast<char**>(&tmp), bytes)) return fail(cuda_status(cudaErrorMemoryAllocation, "temps"));
            cub::DeviceSelect::Flagged(tmp, bytes, iota, fl, sel_eid, nsel, (int)E, s);
        }
        CKS_LAUNCH("rev(select)");
        if (Er > 0) {
            const int rbits = bit_width((uint64_t)n_loc);
            if (!etypes) {
                uint32_t *k0, *k1;
                if (t.alloc(&k0, Er) || t.alloc(&k1, Er)) return fail(cuda_status(cudaErrorMemoryAllocation, "temps"));
                k_rev_keys32<<<grid_for(Er, 256), 256, 0, s>>>(Er, sel_eid, indices, inv_rev, row_begin, k0);
                CKS_LAUNCH("k_rev_keys32");
                CKS(radix_sort_pairs<uint32_t>(t, k0, k1, sel_eid, g->rev.eid, Er, rbits));
            } else {
                uint64_t *k0, *k1;
                if (t.alloc(&k0, Er) || t.alloc(&k1, Er)) return fail(cuda_status(cudaErrorMemoryAllocation, "temps"));
                k_rev_keys64<<<grid_for(Er, 256), 256, 0, s>>>(Er, sel_eid, indices, etypes, inv_rev, row_begin, tbits,
                                                               k0);
                CKS_LAUNCH("k_rev_keys64");
                CKS(radix_sort_pairs<uint64_t>(t, k0, k1, sel_eid, g->rev.eid, Er, rbits + tbits));
                k_gather_i32<<<grid_for(Er, 256), 256, 0, s>>>(Er, g->rev.eid, etypes, g->rev.type);
            }
            k_gather_i32<<<grid_for(Er, 256), 256, 0, s>>>(Er, g->rev.eid, dst, g->rev.nbr);
            CKS_LAUNCH("k_gather(rev)");
        }

        // ---- edge-position map (FWD, or LSF when partitioned) -------------------------------------
        int32_t* pos_of;
        if (t.alloc(&pos_of, E + 1)) return fail(cuda_status(cudaErrorMemoryAllocation, "temps(pos)"));
        if (!part) {
            if (Ef > 0) k_scatter_pos<<<grid_for(Ef, 256), 256, 0, s>>>(Ef, g->fwd.eid, pos_of);
        } else {
            int32_t* cnt;
            if (t.alloc(&cnt, N + 1)) return fail(cuda_status(cudaErrorMemoryAllocation, "temps"));
            cudaMemsetAsync(cnt, 0, sizeof(int32_t) * (N + 1), s);
            if (Er > 0) {
                uint64_t *k0, *k1;
                if (t.alloc(&k0, Er) || t.alloc(&k1, Er)) return fail(cuda_status(cudaErrorMemoryAllocation, "temps"));
                k_dst_keys64<<<grid_for(Er, 256), 256, 0, s>>>(Er, sel_eid, dst, etypes, tbits, k0);
                CKS_LAUNCH("k_dst_keys64");
                CKS(radix_sort_pairs<uint64_t>(t, k0, k1, sel_eid, g->lsf.eid, Er, tbits + bit_width((uint64_t)N)));
                k_scatter_pos<<<grid_for(Er, 256), 256, 0, s>>>(Er, g->lsf.eid, pos_of);
                k_hist_dst<<<grid_for(Er, 256), 256, 0, s>>>(Er, sel_eid, dst, cnt);
            }
            CKS(exclusive_sum(t, cnt, g->lsf.off, N + 1));
        }
        if (Er > 0) k_gather_i32<<<grid_for(Er, 256), 256, 0, s>>>(Er, g->rev.eid, pos_of, g->rev.pos);
        CKS_LAUNCH("pos");

        // ---- R-GCN normaliser 1/c_{v,r} (global, so partitioned ranks see remote destinations) ----
        if (want_norm && E > 0) {
            float* norm_by_eid;
            int32_t* sorted_eid;
            uint64_t *k0, *k1;
            int32_t* iota;
            if (t.alloc(&norm_by_eid, E) || t.alloc(&sorted_eid, E) || t.alloc(&k0, E) || t.alloc(&k1, E) ||
                t.alloc(&iota, E))
                return fail(cuda_status(cudaErrorMemoryAllocation, "temps(norm)"));
            k_iota<<<grid_for(E, 256), 256, 0, s>>>(E, iota);
            k_dst_keys64<<<grid_for(E, 256), 256, 0, s>>>(E, nullptr, dst, etypes, tbits, k0);
            CKS_LAUNCH("k_dst_keys64(norm)");
            CKS(radix_sort_pairs<uint64_t>(t, k0, k1, iota, sorted_eid, E, tbits + bit_width((uint64_t)N)));
            if (etypes) {
                k_rgcn_runs<<<grid_for(N, 128), 128, 0, s>>>(N, indptr, sorted_eid, etypes, norm_by_eid);
            } else {
                int32_t* zeros;
                if (t.alloc(&zeros, E)) return fail(cuda_status(cudaErrorMemoryAllocation, "temps"));
                cudaMemsetAsync(zeros, 0, sizeof(int32_t) * E, s);
                k_rgcn_runs<<<grid_for(N, 128), 128, 0, s>>>(N, indptr, sorted_eid, zeros, norm_by_eid);
            }
            if (Ef > 0) k_gather_f32<<<grid_for(Ef, 256), 256, 0, s>>>(Ef, g->fwd.eid, norm_by_eid, g->fwd.norm);
            if (Er > 0) k_gather_f32<<<grid_for(Er, 256), 256, 0, s>>>(Er, g->rev.eid, norm_by_eid, g->rev.norm);
            CKS_LAUNCH("norm");
        }

        // ---- type-major runs/tasks for the R-GCN weight gradient -----------------------------------
        constexpr int kMeta = 2 * (SEASTAR_NUM_BUCKETS + 1) + 2 + 2 * kPow2Classes;
        long long* d_b;
        if (t.alloc(&d_b, kMeta)) return fail(cuda_status(cudaErrorMemoryAllocation, "temps"));
        cudaMemsetAsync(d_b, 0, sizeof(long long) * kMeta, s);
        long long* d_p2 = d_b + 2 * (SEASTAR_NUM_BUCKETS + 1) + 2;   // [FWD classes | REV classes]
        long long* d_tm = d_b + 2 * (SEASTAR_NUM_BUCKETS + 1);   // [n_runs, n_tasks]
        if (etypes && Ef > 0) {
            const int rbits = bit_width((uint64_t)n_loc);
            int32_t *rowidx, *iota, *tm_pos, *head, *rid, *run_type, *cnt;
            uint64_t *k0, *k1;
            CK(t.alloc(&rowidx, Ef));
            CK(t.alloc(&iota, Ef));
            CK(t.alloc(&tm_pos, Ef));
            CK(t.alloc(&head, Ef));
            CK(t.alloc(&rid, Ef));
            CK(t.alloc(&run_type, Ef));
            CK(t.alloc(&cnt, R + 1));
            CK(t.alloc(&k0, Ef));
            CK(t.alloc(&k1, Ef));
            k_row_index<<<8 * num_sms(), 256, 0, s>>>(n_loc, g->fwd.off, rowidx);
            k_tm_keys<<<grid_for(Ef, 256), 256, 0, s>>>(Ef, rowidx, g->fwd.type, rbits, k0);
            k_iota<<<grid_for(Ef, 256), 256, 0, s>>>(Ef, iota);
            CKS_LAUNCH("k_tm_keys");
            CKS(radix_sort_pairs<uint64_t>(t, k0, k1, iota, tm_pos, Ef, rbits + tbits));
            k_tm_fill<<<grid_for(Ef, 256), 256, 0, s>>>(Ef, tm_pos, g->fwd.nbr, g->fwd.eid, g->fwd.norm, g->tm.src,
                                                        g->tm.eid, g->tm.norm, rowidx, g->fwd.perm, g->tm.dst);
            k_tm_run_heads<<<grid_for(Ef, 256), 256, 0, s>>>(Ef, k1, head);
            CKS_LAUNCH("k_tm_run_heads");
            CKS(inclusive_sum(t, head, rid, Ef));
            k_tm_runs<<<grid_for(Ef, 256), 256, 0, s>>>(Ef, k1, head, rid, rbits, g->fwd.perm, g->tm.run_off,
                                                        g->tm.run_dst, run_type, d_tm);
            k_tm_task_heads<<<grid_for(Ef, 256), 256, 0, s>>>(Ef, d_tm, g->tm.run_off, run_type, kTaskEdges, head);
            CKS_LAUNCH("k_tm_runs");
            CKS(inclusive_sum(t, head, rid, Ef));
            CK(cudaMemsetAsync(cnt, 0, sizeof(int32_t) * (R + 1), s));
            k_tm_tasks<<<grid_for(Ef, 256), 256, 0, s>>>(Ef, d_tm, head, rid, run_type, g->tm.task_run,
                                                         g->tm.task_type, cnt);
            CKS_LAUNCH("k_tm_tasks");
            CKS(exclusive_sum(t, cnt, g->tm.type_task, R + 1));
            // two-phase forward: the same type-major order, with each edge's type and FWD position
            g->fem.nbr = g->tm.src; g->fem.eid = g->tm.eid; g->fem.norm = g->tm.norm; g->fem.n = Ef;
            k_em_type<<<grid_for(Ef, 256), 256, 0, s>>>(Ef, k1, rbits, g->fem.type);
            CK(cudaMemcpyAsync(g->fem.pos, tm_pos, sizeof(int32_t) * Ef, cudaMemcpyDeviceToDevice, s));
            CKS_LAUNCH("k_em_type");
        }
        if (etypes && Er > 0) {
            // REV edges in type-major order (type, rev row, eid) and their segments (two-phase dX)
            const int rbits = bit_width((uint64_t)n_loc);
            int32_t *rowidx, *iota, *pos;
            uint64_t *k0, *k1;
            CK(t.alloc(&rowidx, Er));
            CK(t.alloc(&iota, Er));
            CK(t.alloc(&pos, Er));
            CK(t.alloc(&k0, Er));
            CK(t.alloc(&k1, Er));
            k_row_index<<<8 * num_sms(), 256, 0, s>>>(n_loc, g->rev.off, rowidx);
            k_tm_keys<<<grid_for(Er, 256), 256, 0, s>>>(Er, rowidx, g->rev.type, rbits, k0);
            k_iota<<<grid_for(Er, 256), 256, 0, s>>>(Er, iota);
            CKS_LAUNCH("k_tm_keys(rev)");
            CKS(radix_sort_pairs<uint64_t>(t, k0, k1, iota, pos, Er, rbits + tbits));
            k_tm_fill<<<grid_for(Er, 256), 256, 0, s>>>(Er, pos, g->rev.nbr, g->rev.eid, g->rev.norm, g->rtm_nbr,
                                                        g->rtm_eid, g->rtm_norm);
            CKS_LAUNCH("k_tm_fill(rev)");
            g->rem.nbr = g->rtm_nbr; g->rem.eid = g->rtm_eid; g->rem.norm = g->rtm_norm; g->rem.n = Er;
            k_em_type<<<grid_for(Er, 256), 256, 0, s>>>(Er, k1, rbits, g->rem.type);
            CK(cudaMemcpyAsync(g->rem.pos, pos, sizeof(int32_t) * Er, cudaMemcpyDeviceToDevice, s));
            CKS_LAUNCH("k_em_type(rev)");
        }

        // ---- NEXT-1: local-first splits of FWD and REV (partitioned graphs) -------------------------
        if (part && n_loc > 0) {
            const int rbits1 = bit_width((uint64_t)n_loc) + 1;
            auto split = [&](const IndexSet& x, LocalSplit& sp) -> seastar_status {
                const int64_t ne = x.n_edges;
                SS_CUDA(cudaMemsetAsync(sp.lcnt, 0, sizeof(int32_t) * n_loc, s));
                if (ne == 0) return SEASTAR_OK;
                int32_t *rowidx, *iota, *perm;
                uint64_t *k0, *k1;
                SS_CUDA(t.alloc(&rowidx, ne));
                SS_CUDA(t.alloc(&iota, ne));
                SS_CUDA(t.alloc(&perm, ne));
                SS_CUDA(t.alloc(&k0, ne));
                SS_CUDA(t.alloc(&k1, ne));
                k_row_index<<<8 * num_sms(), 256, 0, s>>>(n_loc, x.off, rowidx);
                k_split_keys<<<grid_for(ne, 256), 256, 0, s>>>(ne, rowidx, x.nbr, row_begin, row_end, k0, sp.lcnt);
                k_iota<<<grid_for(ne, 256), 256, 0, s>>>(ne, iota);
                SS_TRY(check_launch("k_split_keys"));
                SS_TRY(radix_sort_pairs<uint64_t>(t, k0, k1, iota, perm, ne, rbits1));
                k_gather_i32<<<grid_for(ne, 256), 256, 0, s>>>(ne, perm, x.nbr, sp.nbr);
                k_gather_i32<<<grid_for(ne, 256), 256, 0, s>>>(ne, perm, x.eid, sp.eid);
                return check_launch("k_gather(split)");
            };
            CKS(split(g->fwd, g->fsplit));
            CKS(split(g->rev, g->rsplit));
        }

        // ---- a3: degree buckets (second and last sync) --------------------------------------------
        if (n_loc > 0) {
            k_buckets<<<grid_for(n_loc, 256), 256, 0, s>>>(n_loc, g->fwd.off, d_b);
            k_buckets<<<grid_for(n_loc, 256), 256, 0, s>>>(n_loc, g->rev.off, d_b + SEASTAR_NUM_BUCKETS + 1);
            k_pow2_rows<<<grid_for(n_loc, 256), 256, 0, s>>>(n_loc, g->fwd.off, d_p2);
            k_pow2_rows<<<grid_for(n_loc, 256), 256, 0, s>>>(n_loc, g->rev.off, d_p2 + kPow2Classes);
        }
        CKS_LAUNCH("k_buckets");
        long long hb[kMeta];
        cudaMemcpyAsync(hb, d_b, sizeof(hb), cudaMemcpyDeviceToHost, s);
        cudaError_t e = cudaStreamSynchronize(s);
        if (e != cudaSuccess) return fail(cuda_status(e, "graph_create(final)"));
        g->tm.n_runs = hb[2 * (SEASTAR_NUM_BUCKETS + 1)];
        g->tm.n_tasks = hb[2 * (SEASTAR_NUM_BUCKETS + 1) + 1];
        for (int i = 0; i < SEASTAR_NUM_BUCKETS; ++i) {
            g->fwd.bucket_rows[i] = hb[i];
            g->rev.bucket_rows[i] = hb[SEASTAR_NUM_BUCKETS + 1 + i];
        }
        g->fwd.bucket_rows[SEASTAR_NUM_BUCKETS - 1] = n_loc;
        g->rev.bucket_rows[SEASTAR_NUM_BUCKETS - 1] = n_loc;
        for (int i = 0; i < kPow2Classes; ++i) {
            g->fwd.pow2_rows[i] = hb[2 * (SEASTAR_NUM_BUCKETS + 1) + 2 + i];
            g->rev.pow2_rows[i] = hb[2 * (SEASTAR_NUM_BUCKETS + 1) + 2 + kPow2Classes + i];
        }
        g->fwd.max_deg = hb[SEASTAR_NUM_BUCKETS];
        g->rev.max_deg = hb[2 * SEASTAR_NUM_BUCKETS + 1];
    }  // temporaries released (stream-ordered)
    {
        cudaError_t e = cudaStreamSynchronize(s);
        if (e != cudaSuccess) return fail(cuda_status(e, "graph_create(free temps)"));
    }
    *out = g;
    return SEASTAR_OK;
}

seastar_status seastar_graph_destroy(seastar_graph g) {
    if (!g) return SEASTAR_OK;
    int cur = 0;
    cudaGetDevice(&cur);
    if (cur != g->device) cudaSetDevice(g->device);
    cudaError_t e = g->pool ? cudaFree(g->pool) : cudaSuccess;
    if (cur != g->device) cudaSetDevice(cur);
    delete g;
    if (e != cudaSuccess) return cuda_status(e, "graph_destroy");
    return SEASTAR_OK;
}

seastar_status seastar_graph_info(seastar_graph g, seastar_graph_info_t* info) {
    SS_ARG(g && info, "graph_info: NULL argument");
    info->num_nodes = g->N;
    info->num_edges = g->E;
    info->row_begin = g->row_begin;
    info->row_end = g->row_end;
    info->num_fwd_edges = g->fwd.n_edges;
    info->num_rev_edges = g->rev.n_edges;
    info->max_in_degree = g->fwd.max_deg;
    info->max_out_degree = g->rev.max_deg;
    info->num_etypes = g->R;
    info->partitioned = g->partitioned ? 1 : 0;
    for (int i = 0; i < SEASTAR_NUM_BUCKETS; ++i) {
        info->fwd_bucket_rows[i] = g->fwd.bucket_rows[i];
        info->rev_bucket_rows[i] = g->rev.bucket_rows[i];
    }
    return SEASTAR_OK;
}

seastar_status seastar_graph_export(seastar_graph g, int32_t which, int32_t* perm, int32_t* off, int32_t* nbr,
                                    int32_t* eid, int32_t* pos, int32_t* etype, float* norm, seastar_stream stream) {
    SS_ARG(g != nullptr, "graph_export: graph is NULL");
    SS_ARG(which == SEASTAR_FWD || which == SEASTAR_REV || which == SEASTAR_LSF, "graph_export: bad index set %d",
           which);
    SS_ARG(which != SEASTAR_LSF || g->partitioned, "graph_export: LSF exists only for partitioned graphs");
    const IndexSet& x = which == SEASTAR_FWD ? g->fwd : which == SEASTAR_REV ? g->rev : g->lsf;
    SS_ARG(!pos || which == SEASTAR_REV, "graph_export: pos exists only for REV");
    SS_ARG(!etype || x.type, "graph_export: graph is untyped");
    SS_ARG(!norm || x.norm, "graph_export: graph was created without SEASTAR_GRAPH_RGCN_NORM");
    SS_ARG(!(perm && which == SEASTAR_LSF), "graph_export: LSF has no row permutation");
    cudaStream_t s = to_stream(stream);
    auto cp = [&](void* d, const void* src, size_t bytes) -> cudaError_t {
        if (!d || !bytes) return cudaSuccess;
        return cudaMemcpyAsync(d, src, bytes, cudaMemcpyDeviceToDevice, s);
    };
    SS_CUDA(cp(perm, x.perm, sizeof(int32_t) * x.n_rows));
    SS_CUDA(cp(off, x.off, sizeof(int32_t) * (x.n_rows + 1)));
    SS_CUDA(cp(nbr, x.nbr, sizeof(int32_t) * (which == SEASTAR_LSF ? 0 : x.n_edges)));
    SS_CUDA(cp(eid, x.eid, sizeof(int32_t) * x.n_edges));
    SS_CUDA(cp(pos, x.pos, sizeof(int32_t) * x.n_edges));
    SS_CUDA(cp(etype, x.type, sizeof(int32_t) * x.n_edges));
    SS_CUDA(cp(norm, x.norm, sizeof(float) * x.n_edges));
    return SEASTAR_OK;
}

seastar_status seastar_graph_degree_norms(seastar_graph g, int32_t mode, float* src_norm_loc, float* dst_norm_loc,
                                          seastar_stream stream) {
    SS_ARG(g != nullptr, "degree_norms: graph is NULL");
    SS_ARG(mode == SEASTAR_NORM_BOTH || mode == SEASTAR_NORM_IN, "degree_norms: bad mode %d", mode);
    int64_t n = g->n_loc();
    if (n == 0 || (!src_norm_loc && !dst_norm_loc)) return SEASTAR_OK;
    k_degree_norms<<<grid_for(n, 256), 256, 0, to_stream(stream)>>>(n, g->indeg_loc, g->outdeg_loc, mode, src_norm_loc,
                                                                      dst_norm_loc);
    return check_launch("k_degree_norms");
}

}  // extern "C"
