/*
 * seastar.h -- C ABI of the B200-native (sm_100a) Seastar hot path.
 *
 * Seastar (Wu et al., EuroSys'21, /root/reference/PAPER.md) runs GNN layers as fused
 * vertex-centric kernels: per destination vertex over a degree-sorted CSR, gather in-neighbour
 * rows, compute per-edge values, reduce into the vertex's output row (the "Source-Edge-
 * Aggregation" pattern, §6.2), and the symmetric backward over the reverse CSR
 * (§6.3.4).  This header is the whole boundary: plain pointers and sizes, no torch
 * types.  A thin Python binding with the same names sits above it
 * (paper_conf_eurosys_wumcjlzcy21_b200/_lib.py).
 *
 * Conventions (apply to every entry point)
 *   * Pointers marked "dev" are CUDA device pointers on the current device; "host" are host
 *     pointers.  All feature/parameter/gradient/workspace buffers are owned by the caller; the
 *     graph handle owns only its internal index arrays.
 *   * Dense matrices are row-major fp32 with an explicit leading dimension (row stride, in
 *     elements) `ld >= width`.  When `ld % 4 == 0` and the base pointer is 16-byte aligned the
 *     kernels use 128-bit loads; otherwise they fall back to 32-bit loads (same results).
 *   * "_all" arrays cover all N vertices (after the caller's all-gather when the graph is
 *     partitioned); "_loc" arrays cover the owned vertex range [row_begin,row_end) and are indexed
 *     by (v - row_begin).  On one GPU row_begin = 0, row_end = N and both are the same.
 *   * Every call is asynchronous and stream-ordered on `stream` (a cudaStream_t; NULL = legacy
 *     default stream) except seastar_graph_create, which synchronises once.  Nothing allocates
 *     device memory except seastar_graph_create.  All calls are capturable in a CUDA graph except
 *     seastar_graph_create/destroy.
 *   * Errors: every entry returns a seastar_status and never throws.  Arguments are validated
 *     before any launch (no partial writes on INVALID_ARGUMENT).  seastar_last_error() returns a
 *     thread-local message for the last failure.  Asynchronous kernel faults surface as
 *     SEASTAR_ERR_CUDA on a later call.  Devices other than sm_100 get SEASTAR_ERR_UNSUPPORTED;
 *     there is no CPU fallback.
 *   * Forward kernels use no atomics and fixed reduction trees: results are bitwise
 *     deterministic run to run.
 */
#ifndef SEASTAR_H_
#define SEASTAR_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SEASTAR_ABI_VERSION 2

typedef struct seastar_graph_s* seastar_graph;   /* opaque, immutable after create */
/* NEXT-3 dropout descriptor (reading #27): drop probability p (0 <= p < 1), the mask's site id
 * and seed, and a device int32 step counter (or NULL = 0) read on the device so a captured CUDA graph draws a
 * fresh mask every epoch.  keep(i) <=> (sm64(key ^ i) >> 40) >= round(p * 2^24),
 * key = sm64(seed ^ sm64((site << 32) | step)), sm64 = splitmix64's output function. */
typedef struct {
    float p;
    uint32_t site;
    uint64_t seed;
    const int32_t* step;
} seastar_dropout_spec;
typedef void* seastar_stream;                     /* cudaStream_t */

typedef enum {
    SEASTAR_OK = 0,
    SEASTAR_ERR_INVALID_ARGUMENT = 1,
    SEASTAR_ERR_INVALID_GRAPH = 2,
    SEASTAR_ERR_OUT_OF_MEMORY = 3,
    SEASTAR_ERR_CUDA = 4,
    SEASTAR_ERR_UNSUPPORTED = 5
} seastar_status;

/* activation g(.) of Eq. 1; derivatives are taken from the output Y */
typedef enum {
    SEASTAR_ACT_NONE = 0,
    SEASTAR_ACT_RELU = 1,
    SEASTAR_ACT_ELU = 2,      /* alpha = 1 */
    SEASTAR_ACT_SIGMOID = 3
} seastar_act;

/* graph_create flags */
#define SEASTAR_GRAPH_RGCN_NORM 1u   /* precompute the R-GCN normaliser 1/c_{v,r} per edge */

/* index sets exported by seastar_graph_export */
#define SEASTAR_FWD 0   /* in-edges of owned rows, rows sorted by in-degree desc (Fig. 7 "CSR")           */
#define SEASTAR_REV 1   /* out-edges of owned rows, rows sorted by out-degree desc (Fig. 7 "Reversed CSR") */
#define SEASTAR_LSF 2   /* partitioned graphs only: edges with owned source grouped by dst id */

/* degree-norm modes for seastar_graph_degree_norms */
#define SEASTAR_NORM_BOTH 0   /* src_norm = outdeg^-1/2, dst_norm = indeg^-1/2 (GCN, DGL norm='both') */
#define SEASTAR_NORM_IN 1     /* src_norm = dst_norm = indeg^-1/2 (APPNP, DGL APPNPConv)               */

/* Degree classes (a3): rows whose degree is >= threshold[i] form a prefix of the sorted rows. */
#define SEASTAR_NUM_BUCKETS 4
/* thresholds: 1024 (hub), 32 (warp per row), 1 (sub-warp group per row), 0 (empty rows) */

typedef struct {
    int64_t num_nodes;          /* N */
    int64_t num_edges;          /* E */
    int64_t row_begin, row_end; /* owned vertex range */
    int64_t num_fwd_edges;      /* in-edges of owned rows */
    int64_t num_rev_edges;      /* out-edges of owned rows */
    int64_t max_in_degree;      /* over owned rows */
    int64_t max_out_degree;     /* over owned rows */
    int32_t num_etypes;         /* R (1 for untyped graphs) */
    int32_t partitioned;        /* 1 if [row_begin,row_end) != [0,N) (LSF index present) */
    int64_t fwd_bucket_rows[SEASTAR_NUM_BUCKETS]; /* # fwd rows with in-degree  >= 1024, 32, 1, 0 */
    int64_t rev_bucket_rows[SEASTAR_NUM_BUCKETS]; /* # rev rows with out-degree >= 1024, 32, 1, 0 */
} seastar_graph_info_t;

/* ------------------------------------------------------------------------------------------ */
/* library                                                                                     */
/* ------------------------------------------------------------------------------------------ */
const char* seastar_last_error(void);   /* thread-local; valid until the next failing call */
int32_t seastar_abi_version(void);       /* SEASTAR_ABI_VERSION */
/* 0 if the current device is sm_100 (B200) and the kernels are loadable, else UNSUPPORTED/CUDA */
seastar_status seastar_device_check(void);

/* ------------------------------------------------------------------------------------------ */
/* a1-a3: graph representation (§6.1, Fig. 7, §6.3.3, §6.3.4, */
/* §6.3.5)                                                                           */
/* ------------------------------------------------------------------------------------------ */
/*
 * Build the degree-sorted forward CSR, the reverse CSR with carried edge ids, the edge-position
 * map and the degree buckets for the owned vertex range [row_begin,row_end).
 *   N, E          : vertices and edges; 0 <= N < 2^31, 0 <= E < 2^31.
 *   indptr  (dev) : [N+1] int64 user in-CSR offsets (monotone, indptr[0]=0, indptr[N]=E).
 *   indices (dev) : [E] int64 source vertex ids; edge e is the e-th entry (user edge id = e),
 *                   its destination is the row containing it.
 *   etypes  (dev) : [E] int32 edge types in [0,num_etypes), or NULL (untyped, num_etypes ignored).
 *   row_begin/end : owned destination/source range, 0 <= row_begin <= row_end <= N.
 *   flags         : SEASTAR_GRAPH_RGCN_NORM or 0.
 * Order (pinned by Fig. 7): fwd rows by (in-degree desc, id asc); rev rows by (out-degree desc,
 * id asc); edges inside a row by (type asc, eid asc).  The input arrays are only read; the
 * handle owns copies in int32.  Invalid contents -> SEASTAR_ERR_INVALID_GRAPH.  Synchronises
 * `stream` once (reads back the validation flag and bucket sizes).
 */
seastar_status seastar_graph_create(int64_t N, int64_t E, const int64_t* indptr, const int64_t* indices,
                                    const int32_t* etypes, int32_t num_etypes, int64_t row_begin,
                                    int64_t row_end, uint32_t flags, seastar_stream stream,
                                    seastar_graph* out);
seastar_status seastar_graph_destroy(seastar_graph g);
seastar_status seastar_graph_info(seastar_graph g, seastar_graph_info_t* info /* host */);
/*
 * Copy one index set to caller buffers (dev; any may be NULL):
 *   FWD: perm[n_loc] (row -> vertex), off[n_loc+1], nbr[E_fwd] (src ids), eid, etype, norm (RGCN);
 *   REV: perm[n_loc], off[n_loc+1], nbr[E_rev] (dst ids), eid, pos (position of the edge in FWD,
 *        or in LSF when partitioned), etype, norm;
 *   LSF: perm = NULL, off[N+1] by dst id, eid[E_rev].
 */
seastar_status seastar_graph_export(seastar_graph g, int32_t which, int32_t* perm, int32_t* off, int32_t* nbr,
                                    int32_t* eid, int32_t* pos, int32_t* etype, float* norm,
                                    seastar_stream stream);
/* per-owned-vertex degree norms deg^-1/2 (deg clamped >= 1), [n_loc] each (dev; either may be NULL) */
seastar_status seastar_graph_degree_norms(seastar_graph g, int32_t mode, float* src_norm_loc,
                                          float* dst_norm_loc, seastar_stream stream);

/* ------------------------------------------------------------------------------------------ */
/* a4 / a11: dense per-layer transform (the unfused S-type ops of PAPER.md L289; Fig. 2 f = W h) */
/* ------------------------------------------------------------------------------------------ */
/*
 * Y[r,:] = row_scale[r] * act(X[r,:] W + bias)      for r < M
 *   X (dev) [M,K] ld ldx ; W (dev) [K,Nout] row-major (ld Nout) ; bias [Nout] or NULL ;
 *   row_scale [M] or NULL ; Y (dev) [M,Nout] ld ldy.  fp32 in / out, fp32-accurate.
 * With a workspace of seastar_linear_fwd_workspace(K, Nout) bytes, ldx % 4 == 0, a 16-byte aligned X,
 * M >= 128, K >= 32 and Nout <= 128 it runs on the tcgen05 tensor cores (TMA-fed, TMEM accumulators,
 * 3xTF32 hi/lo split: W is split once per call into the workspace); otherwise a SIMT fp32 kernel.
 */
seastar_status seastar_linear_fwd(const float* X, int64_t M, int64_t K, int64_t ldx, const float* W,
                                  int64_t Nout, const float* bias, const float* row_scale, seastar_act act,
                                  float* Y, int64_t ldy, void* workspace, size_t ws_bytes, seastar_stream stream);
size_t seastar_linear_fwd_workspace(int64_t K, int64_t Nout);
/*
 * dX[r,:] = row_scale[r] * (dY[r,:] W^T) * act'(Yact[r,:])
 *   dY [M,Nout] ld ldy ; W [K,Nout] row-major ; row_scale [M] or NULL ; Yact [M,K] ld ldx or NULL (the
 *   activation output of the layer below, so the activation backward is fused) ; dX [M,K] ld ldx.
 */
seastar_status seastar_linear_bwd_data(const float* dY, int64_t M, int64_t Nout, int64_t ldy, const float* W,
                                       int64_t K, const float* row_scale, const float* Yact, seastar_act act,
                                       float* dX, int64_t ldx, seastar_stream stream);
/*
 * dW = X^T dY  ([K,Nout], any Nout >= 1, produced in column chunks of 64) and, if db != NULL,
 * db = sum_r dY[r,:].  Deterministic split-M reduction through `workspace` (dev) of
 * seastar_linear_bwd_weight_workspace() bytes; the split partials are summed in split order with an
 * fp64 accumulator.
 */
seastar_status seastar_linear_bwd_weight(const float* X, int64_t M, int64_t K, int64_t ldx, const float* dY,
                                         int64_t Nout, int64_t ldy, float* dW, float* db, void* workspace,
                                         size_t ws_bytes, seastar_stream stream);
size_t seastar_linear_bwd_weight_workspace(int64_t M, int64_t K, int64_t Nout);

/* ------------------------------------------------------------------------------------------ */
/* a5 / a8: GCN and APPNP aggregation (Fig. 1 L85-L93, Fig. 3, Alg. 1,  */
/* §6.3.2; backward on the reverse CSR §6.3.4)                                   */
/* ------------------------------------------------------------------------------------------ */
/*
 * For every owned vertex v (fused: gather -> sum -> epilogue, one pass over in(v)):
 *   z     = dst_norm[v] * sum_{e in in(v)} T_all[src(e),:]          (T_all already src-scaled)
 *   z     = (1 - alpha) * z + alpha * H0_loc[v]                       if H0_loc != NULL (APPNP)
 *   Y[v]  = act(z + bias)                                             (bias NULL -> 0)
 *   Ys[v] = out_scale[v] * Y[v]                                       if Ys_loc != NULL
 * T_all [N,F] ld ld; dst_norm/out_scale [n_loc] or NULL; H0_loc, Y_loc, Ys_loc [n_loc,F] ld ld.
 */
seastar_status seastar_gcn_fwd(seastar_graph g, const float* T_all, int64_t F, int64_t ld, const float* dst_norm,
                               const float* bias, seastar_act act, float alpha, const float* H0_loc,
                               float* Y_loc, const float* out_scale, float* Ys_loc,
                               const seastar_dropout_spec* edge_drop, seastar_stream stream);
/* (edge_drop: NULL, or NEXT-3 edge dropout (DGL APPNPConv edge_drop): edge e's message is multiplied by
 *  keep(eid) / (1 - p), eid = user edge id; the backward takes the same spec) */
/*
 * Adjoint over the reverse CSR, for every owned vertex u:
 *   g       = scale * src_norm[u] * sum_{e in out(u)} dP_all[dst(e),:]
 *   g       = g * act'(Yact_loc[u])                                   if Yact_loc != NULL (act' from Y)
 *   dA[u]   = g                                                       if dA_loc != NULL
 *   dP[u]   = post_scale[u] * g                                       if dP_loc != NULL
 * dP_all [N,F] ld ld (= dst_norm * upstream gradient, gathered); src_norm/post_scale [n_loc] or NULL.
 * At least one of dA_loc / dP_loc must be non-NULL.
 */
seastar_status seastar_gcn_bwd(seastar_graph g, const float* dP_all, int64_t F, int64_t ld, const float* src_norm,
                               float scale, const float* Yact_loc, seastar_act act, const float* post_scale,
                               float* dA_loc, float* dP_loc, const seastar_dropout_spec* edge_drop,
                               seastar_stream stream);
/*
 * NEXT-1 (multi-GPU overlap): seastar_gcn_fwd / seastar_gcn_bwd of a row-partitioned graph in two
 * phases around the all-gather of the source table.  graph_create keeps, per owned row, its edges re-ordered with
 * the edges whose neighbour is an owned vertex first.
 *   phase 1: part[v, :F] = sum over the owned-neighbour edges of the row, read from the rank's OWN rows (T_loc /
 *            dP_loc_in [n_loc, F] ld ldloc, row i = vertex row_begin + i) -- it needs no gathered data, so it runs
 *            while the all-gather is in flight; no epilogue.  T_all / dP_all and the outputs are ignored.
 *   phase 2: the remaining edges from the gathered table (T_all / dP_all), + part, then the same epilogue as
 *            seastar_gcn_fwd / seastar_gcn_bwd (all their arguments keep their meaning).  T_loc is ignored.
 *   part: [n_loc, F] ld ldp (dev, caller-owned scratch, written by phase 1 and read by phase 2).
 * The sum is taken in (owned part, rest) order: deterministic, and within the tolerance of the one-phase call
 * (the order of a row's terms differs).  INVALID_ARGUMENT for an unpartitioned graph.
 */
seastar_status seastar_gcn_fwd_split(seastar_graph g, int32_t phase, const float* T_loc, int64_t ldloc,
                                     const float* T_all, int64_t F, int64_t ld, const float* dst_norm,
                                     const float* bias, seastar_act act, float alpha, const float* H0_loc,
                                     float* Y_loc, const float* out_scale, float* Ys_loc, float* part, int64_t ldp,
                                     const seastar_dropout_spec* edge_drop, seastar_stream stream);
seastar_status seastar_gcn_bwd_split(seastar_graph g, int32_t phase, const float* dP_loc_in, int64_t ldloc,
                                     const float* dP_all, int64_t F, int64_t ld, const float* src_norm, float scale,
                                     const float* Yact_loc, seastar_act act, const float* post_scale, float* dA_loc,
                                     float* dP_loc, float* part, int64_t ldp, const seastar_dropout_spec* edge_drop,
                                     seastar_stream stream);

/* ------------------------------------------------------------------------------------------ */
/* a6 / a9: GAT (Fig. 2 L95-L123, Fig. 3, FSM units L391-L393)                   */
/* ------------------------------------------------------------------------------------------ */
/* el[u,h] = <T[u,h,:], a_l[h,:]>, er[u,h] = <T[u,h,:], a_r[h,:]>   (T [M,H*F] ld ldt; el/er [M,H]) */
seastar_status seastar_gat_attn_proj(const float* T, int64_t M, int32_t H, int32_t F, int64_t ldt, const float* a_l,
                                     const float* a_r, float* el, float* er, seastar_stream stream);
/*
 * Fused forward, one pass over in(v) with an online softmax per head:
 *   s_e = el_all[src(e),h] + er_loc[v,h];  z_e = LeakyReLU_slope(s_e);
 *   A[v,h,:] = sum_e softmax_e(z) T_all[src(e),h,:]  (0 for an empty row);
 *   lse[v,h] = log sum_e exp(z_e) (-inf for an empty row);  Y[v] = act(A[v] + bias).
 * Optional (B_loc and b_loc both non-NULL): from the same gathered rows also
 *   B[v,h,:] = sum_e a_e LeakyReLU'(s_e) T_all[src(e),h,:]   and   b[v,h] = sum_e a_e LeakyReLU'(s_e),
 * the forward-only factors of der_v = sum_e ds_e = <dA_v, B_v> - c_v b_v, so that the backward needs no
 * destination-major edge pass (seastar_gat_bwd_prep then emits der directly).
 * T_all [N,H*F] ld ldt ; el_all [N,H] ; er_loc/lse_loc/b_loc [n_loc,H] ; A_loc, Y_loc, B_loc [n_loc,H*F] ld ldt.
 * Requires F % 4 == 0 or H == 1 for the 128-bit path (otherwise 32-bit loads are used).
 */
seastar_status seastar_gat_fwd(seastar_graph g, const float* T_all, const float* el_all, const float* er_loc,
                               int32_t H, int32_t F, int64_t ldt, float slope, const float* bias, seastar_act act,
                               float* A_loc, float* Y_loc, float* lse_loc, float* B_loc, float* b_loc,
                               const seastar_dropout_spec* attn_drop, seastar_stream stream);
/* (attn_drop: NULL, or NEXT-3 attention dropout -- see seastar_dropout_spec; the aggregation uses
 *  a_e * m_e with m_e = keep(eid * H + h) / (1 - p), the softmax and lse are not masked.  With p > 0 the
 *  generic chunked kernels run (H*F <= 128).  gat_bwd and gat_der must get the same spec.) */
/* leading dimension (floats) of the packed per-destination backward record D: round_up(H*F, 4) + 4*H */
int64_t seastar_gat_record_ld(int32_t H, int32_t F);
/*
 * Backward row pass over owned rows: dA = dY * act'(Y);  c[v,h] = <dA[v,h,:], A[v,h,:]>;
 * D_loc[v] = [ dA (H*F, zero-padded to a multiple of 4) | per head (er, lse, c, nl2) ],
 * nl2 = -lse * log2(e) (the backward kernels form a_e = 2^(LeakyReLU(s_e) log2(e) + nl2))
 * (ld = seastar_gat_record_ld(H,F); every field is 16-byte aligned when D_loc is).
 * If B_loc, b_loc (saved by seastar_gat_fwd) and der_loc [n_loc,H] are given, also
 *   der_loc[v,h] = <dA[v,h,:], B[v,h,:]> - c[v,h] b[v,h]    (replaces seastar_gat_der).
 */
seastar_status seastar_gat_bwd_prep(seastar_graph g, const float* dY_loc, const float* Y_loc, seastar_act act,
                                    const float* A_loc, const float* er_loc, const float* lse_loc, int32_t H,
                                    int32_t F, int64_t ldt, float* D_loc, const float* B_loc, const float* b_loc,
                                    float* der_loc, seastar_stream stream);
/*
 * Fused source-major backward over the reverse CSR, for every owned u and out-edge e = (u -> v):
 *   a_e = exp(LeakyReLU(el[u,h] + er[v,h]) - lse[v,h]);  g_e = <dA[v,h,:], T[u,h,:]>;
 *   ds_e = a_e (g_e - c[v,h]) LeakyReLU'(s_e);
 *   dT_loc[u,h,:] = sum_e a_e dA[v,h,:];  del_loc[u,h] = sum_e ds_e   (registers, no atomics).
 * T_loc [n_loc,H*F] ld ldt; el_loc [n_loc,H]; D_all [N, gat_record_ld] (gathered records).
 */
seastar_status seastar_gat_bwd(seastar_graph g, const float* T_loc, const float* el_loc, const float* D_all,
                               int32_t H, int32_t F, int64_t ldt, float slope, float* dT_loc, float* del_loc,
                               const seastar_dropout_spec* attn_drop, seastar_stream stream);
/*
 * Fused destination-major pass over the forward CSR: der_loc[v,h] = sum_{e in in(v)} ds_e with ds_e
 * recomputed from the gathered T_all / el_all rows and v's own record D_loc[v] (no E x H array is
 * materialised; when partitioned each rank computes its owned rows, no reduction is needed).
 * T_all [N,H*F] ld ldt, el_all [N,H] (the forward's gathered tables); D_loc [n_loc, gat_record_ld];
 * der_loc [n_loc,H].
 */
seastar_status seastar_gat_der(seastar_graph g, const float* T_all, const float* el_all, const float* D_loc,
                               int32_t H, int32_t F, int64_t ldt, float slope, float* der_loc,
                               const seastar_dropout_spec* attn_drop, seastar_stream stream);
/*
 * Backward of seastar_gat_attn_proj over M rows:  dT[u,h,:] += del[u,h] a_l[h,:] + der[u,h] a_r[h,:];
 * da_l = sum_u del[u,h] T[u,h,:];  da_r = sum_u der[u,h] T[u,h,:]   (deterministic, via workspace of
 * seastar_gat_attn_proj_bwd_workspace() bytes).  del/der may be NULL (treated as 0).
 */
seastar_status seastar_gat_attn_proj_bwd(const float* T, int64_t M, int32_t H, int32_t F, int64_t ldt,
                                         const float* a_l, const float* a_r, const float* del, const float* der,
                                         float* dT, float* da_l, float* da_r, void* workspace, size_t ws_bytes,
                                         seastar_stream stream);
size_t seastar_gat_attn_proj_bwd_workspace(int64_t M, int32_t H, int32_t F);

/* ------------------------------------------------------------------------------------------ */
/* a7 / a10: R-GCN (§6.3.5: outer loop over types unrolled by detecting type */
/* changes in the type-sorted edge list)                                                       */
/* ------------------------------------------------------------------------------------------ */
/*
 * Y[v] = act( sum_r ( sum_{e in in(v), type(e)=r} norm_e X_all[src(e),:] ) W[r] + bias )
 *   X_all [N,F_in] ld ldx ; W [R,F_in,F_out] ; norm_user [E] by user edge id, or NULL = the
 *   graph's 1/c_{v,r} (requires SEASTAR_GRAPH_RGCN_NORM) ; Y_loc [n_loc,F_out] ld ldy.
 *   F_in, F_out <= 64.
 *   Three paths, chosen by shape (all deterministic; no floating-point atomics):
 *   - default when F_in, F_out <= 16 (every R-GCN layer of the BASELINE configs; rgcn_tile.cu): edge-balanced
 *     tiles of 512 edges in row order; each tile's gathered rows are staged in shared memory, its edges grouped by
 *     type with a shared-memory counting sort, every edge's product norm_e X_all[src(e)] W[type(e)] computed with
 *     the W[type] column held in registers across a type run, then each row sums its products in row order
 *     ((type, eid) order); a row cut by tile borders is summed over its tiles in tile order.  W is resident in
 *     shared memory ([R][16][round4(F_in)] fp32, persistent CTAs) when R * 64 * round4(F_in) + 82 KB fits in
 *     227 KB, else read through L1/L2 (one tile per CTA).  workspace: seastar_rgcn_fwd_workspace() bytes
 *     (dev, caller-owned: 128 B per tile, contents undefined on return); INVALID_ARGUMENT if it is smaller.
 *     SEASTAR_RGCN_ROWS=1 selects the one-pass path below instead.
 *   - opt-in (environment SEASTAR_RGCN_TWOPHASE=1), F_in, F_out <= 16 and R * F_in * round4(F_out) * 4 <=
 *     200 KB (two-phase; slower than the one pass on the AM shape, kept for the r2 measurements): the edges are visited in
 *     type-major order, a lane per edge, with W staged in shared memory (the 32 edges of a warp share their
 *     type, so every W read is a broadcast); edge e's product norm_e X_all[src(e)] W[type(e)] goes to slot e
 *     of `workspace` in row order, and each row sums its slots in (type, eid) order.  workspace:
 *     seastar_rgcn_fwd_workspace() bytes (dev, caller-owned, contents undefined on return); INVALID_ARGUMENT
 *     if it is smaller.
 *   - otherwise (one pass; PAPER.md L473-L475 as written): every row walks its type-sorted edges and flushes
 *     each run through W[r] staged in shared memory (stride S floats per W[r]: the smallest stride
 *     >= F_in * round4(F_out) that is 16 mod 32 if R * S * 4 <= 219 KB, else the dense F_in * round4(F_out));
 *     needs R * S * 4 <= 227 KB - 256 B, and <= 219 KB when some row has degree >= 1024 (the hub CTAs keep an
 *     8 KB reduction buffer); UNSUPPORTED beyond.  seastar_rgcn_fwd_workspace() returns 0 (workspace may be NULL).
 *   The workspace of seastar_rgcn_fwd_workspace() covers the path the library will take for this shape.
 */
seastar_status seastar_rgcn_fwd(seastar_graph g, const float* X_all, int64_t F_in, int64_t ldx, const float* W,
                                int64_t F_out, const float* norm_user, const float* bias, seastar_act act,
                                float* Y_loc, int64_t ldy, void* workspace, size_t ws_bytes, seastar_stream stream);
size_t seastar_rgcn_fwd_workspace(seastar_graph g, int64_t F_in, int64_t F_out);
/*
 * Backward of seastar_rgcn_fwd's pre-activation output given dA = dL/d(pre-activation):
 *   dX_loc[u] = sum_{type runs r of out(u)} (sum_{e in run} norm_e dA_all[dst(e),:]) W[r]^T
 *     -- source-major over the type-sorted reverse CSR (§6.3.4 L461 + §6.3.5);
 *   dW[r] = sum_{owned v} g_{v,r}^T dA_all[v,:],  g_{v,r} = sum_{e in in(v), type r} norm_e X_all[src(e),:]
 *     -- over a type-major view of the forward edges built at graph_create, cut into tasks of one type; per task
 *     (F_in, F_out <= 16) the rows X_all[src] and dA_all[dst] are staged in shared memory and every warp keeps its
 *     dW_r partial in registers, summing the per-edge outer products norm_e X_all[src]^T dA_all[dst]; partials
 *     are reduced per type in task order (deterministic).
 *   X_all [N,F_in] ld ldx (the forward's gathered input) ; dA_all [N,F_out] ld ldd (gathered) ;
 *   dX_loc [n_loc,F_in] ld ldx or NULL ; dW [R,F_in,F_out] or NULL (overwritten; this rank's partial
 *   when partitioned).  ldx, ldd multiples of 4; F_in*F_out <= 1024.
 *   workspace: seastar_rgcn_bwd_workspace() bytes (dev).
 */
seastar_status seastar_rgcn_bwd(seastar_graph g, const float* X_all, int64_t F_in, int64_t ldx,
                                const float* dA_all, int64_t F_out, int64_t ldd, const float* W,
                                const float* norm_user, const float* Yact_loc, seastar_act act, float* dX_loc,
                                float* dW, void* workspace, size_t ws_bytes, seastar_stream stream);
/* (Yact_loc [n_loc,F_in] ld ldx or NULL: dX_loc is multiplied by act'(Yact_loc), fusing the input
 *  layer's activation backward; act is ignored when Yact_loc is NULL.  dX takes the path seastar_rgcn_fwd would
 *  take over the reverse edges (tile by default for F_in, F_out <= 16); the workspace covers dX and dW.) */
size_t seastar_rgcn_bwd_workspace(seastar_graph g, int64_t F_in, int64_t F_out);

/* ------------------------------------------------------------------------------------------ */
/* NEXT-2: R-GCN as the paper ran it -- featureless input layer, basis decomposition            */
/* (Table 2 L485 / Table 3 L1219-L1227 aifb, mutag, bgs; layer of [53]; DESIGN.md      */
/* reading #26).  W_r = sum_b a[r,b] V_b ; featureless h_u = one-hot(u) => h_u W_r = sum_b a[r,b] V[u,b,:]. */
/* ------------------------------------------------------------------------------------------ */
/*
 * Y[v] = act( sum_{e in in(v)} norm_e sum_b a[type(e),b] V_all[src(e), b*F : b*F+F] + loop[v] + bias )
 *   V_all [N, B*F] ld ldv (dev; row u = the B basis rows of vertex u, basis-major; gathered by source
 *   id, so a partitioned caller all-gathers it) ; a [R, B] (dev) ; norm_user [E] by user edge id or NULL
 *   = the graph's 1/c_{v,r} ; loop_loc [n_loc, F] ld ldl or NULL (self-loop addend, e.g. W_0[v] of a
 *   featureless self-loop) ; bias [F] or NULL ; Y_loc [n_loc, F] ld ldy.
 *   F a power of two in [4, 128]; B*F <= 2048; R*B*4 <= 96 KB; ldv, ldy multiples of 4, pointers 16B aligned.
 *   One warp per destination row, no atomics (bitwise deterministic).
 */
seastar_status seastar_rgcn_basis_fwd(seastar_graph g, const float* V_all, int64_t B, int64_t F, int64_t ldv,
                                      const float* a, const float* norm_user, const float* loop_loc, int64_t ldl,
                                      const float* bias, seastar_act act, float* Y_loc, int64_t ldy,
                                      seastar_stream stream);
/*
 * VJP of seastar_rgcn_basis_fwd's pre-activation output given dA_all = dL/d(pre-activation) [N, F] ld ldd
 * (gathered by destination id):
 *   dV_loc[u, b*F + f] = sum_{e in out(u)} norm_e a[type(e),b] dA_all[dst(e), f]   (owned sources u;
 *     source-major over the reverse CSR, no atomics) -- NULL to skip ;
 *   da[r, b] = sum_{e: type(e)=r} norm_e <V_all[src(e), b*F : b*F+F], dA_all[dst(e), :]>  (over the
 *     type-major view built at graph_create; per-task partials reduced per type in task order in
 *     fp64; this rank's partial when partitioned) -- NULL to skip.
 *   The self-loop and bias gradients are dA itself and its column sum (the caller's).
 *   dV_loc [n_loc, B*F] ld ldv ; workspace: seastar_rgcn_basis_bwd_workspace() bytes when da != NULL.
 */
seastar_status seastar_rgcn_basis_bwd(seastar_graph g, const float* V_all, int64_t B, int64_t F, int64_t ldv,
                                      const float* a, const float* norm_user, const float* dA_all, int64_t ldd,
                                      float* dV_loc, float* da, void* workspace, size_t ws_bytes,
                                      seastar_stream stream);
size_t seastar_rgcn_basis_bwd_workspace(seastar_graph g, int64_t B);
/*
 * Basis combination for a dense R-GCN layer: W[r, k] = sum_b a[r,b] Vb[b, k] for k < K
 * (a [R,B], Vb [B,K], W [R,K], all dev, contiguous; K = F_in*F_out of seastar_rgcn_fwd's W).
 * fp64 accumulation in a fixed order.
 */
seastar_status seastar_basis_combine(const float* a, const float* Vb, int32_t R, int32_t B, int64_t K, float* W,
                                     seastar_stream stream);
/* its VJP: da[r,b] = <dW[r,:], Vb[b,:]>, dVb[b,k] = sum_r a[r,b] dW[r,k]; either output may be NULL */
seastar_status seastar_basis_combine_bwd(const float* a, const float* Vb, const float* dW, int32_t R, int32_t B,
                                         int64_t K, float* da, float* dVb, seastar_stream stream);

/* ------------------------------------------------------------------------------------------ */
/* training-step glue kept on the GPU (DGL default loop)                         */
/* ------------------------------------------------------------------------------------------ */
/*
 * Softmax cross-entropy over this rank's M rows, normalised by the global row count n_total (>= M;
 * = M on one GPU) so that per-rank gradients all-reduce to the full-batch gradient:
 *   loss (dev scalar) = sum_r (lse(Z_r) - Z_r[label_r]) / n_total ;  dZ = (softmax(Z) - onehot) / n_total.
 * Z [M,C] ld ldz, labels (dev) [M] int64, dZ [M,C] ld lddz or NULL.
 * workspace: seastar_softmax_xent_workspace() bytes.
 */
seastar_status seastar_softmax_xent(const float* Z, int64_t M, int64_t n_total, int32_t C, int64_t ldz,
                                    const int64_t* labels, float* loss, float* dZ, int64_t lddz, void* workspace,
                                    size_t ws_bytes, seastar_stream stream);
size_t seastar_softmax_xent_workspace(int64_t M);
/* out[j] = sum_r X[r,j] for j < F (deterministic two-stage), workspace: seastar_colsum_workspace() */
seastar_status seastar_colsum(const float* X, int64_t M, int64_t F, int64_t ld, float* out, void* workspace,
                              size_t ws_bytes, seastar_stream stream);
size_t seastar_colsum_workspace(int64_t M, int64_t F);
/* y = a * x + b * y over n floats */
seastar_status seastar_axpby(int64_t n, float a, const float* x, float b, float* y, seastar_stream stream);
/* Y[i, :F] = scale[i] * X[i, :F] for i < M (dev; ldx, ldy >= F; Y may alias X) -- the APPNP propagation's
 * n (.) pre-scaling of a table (reading #23), without a dense transform */
seastar_status seastar_row_scale(const float* X, int64_t M, int64_t F, int64_t ldx, const float* scale, float* Y,
                                 int64_t ldy, seastar_stream stream);
/*
 * One Adam step over a flat parameter buffer (Kingma & Ba Alg. 1), step number read from
 * *step (dev int32, >= 1) so the call can be captured in a CUDA graph; see seastar_step_inc.
 */
seastar_status seastar_adam(float* param, const float* grad, float* m, float* v, int64_t n, float lr, float beta1,
                            float beta2, float eps, const int32_t* step, seastar_stream stream);
/*
 * NEXT-3: reproducible inverted dropout ("a Dropout layer"; DGL default configs L481;
 * DESIGN.md reading #27).  Y[r,f] = keep(i) ? X[r,f] / (1 - p) : 0 with i = (row0 + r) * F + f (the
 * element's GLOBAL index, so a row-partitioned caller passes row0 = row_begin and reproduces the
 * single-GPU mask) and
 *   key = sm64(seed ^ sm64((site << 32) | step)),  keep(i) <=> (sm64(key ^ i) >> 40) >= round(p * 2^24),
 * sm64 = splitmix64's output function.  `step` (dev int32, e.g. the Adam step counter) or NULL (= 0) is
 * read on the device, so a captured CUDA graph draws a fresh mask every epoch.  The mask is a pure
 * function of (seed, site, step, i): the backward is the same call on dY.  X [M,F] ld ldx, Y [M,F] ld
 * ldy (dev; Y == X allowed when ldy == ldx).  0 <= p < 1.
 */
seastar_status seastar_dropout(const float* X, int64_t M, int64_t F, int64_t ldx, int64_t row0, float p, uint64_t seed,
                               uint32_t site, const int32_t* step, float* Y, int64_t ldy, seastar_stream stream);
/* *counter += 1 on the device */
seastar_status seastar_step_inc(int32_t* counter, seastar_stream stream);

#ifdef __cplusplus
}
#endif
#endif /* SEASTAR_H_ */
