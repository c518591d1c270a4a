/*
 * seastar_oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously-correct CPU implementation of what Seastar's hot path computes
 * (Wu et al., "Seastar: Vertex-Centric Programming for Graph Neural Networks", EuroSys'21,
 * /root/reference/PAPER.md).  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load it.  It shares no code with the CUDA path
 * (paper_conf_eurosys_wumcjlzcy21_b200/csrc) and includes none of its headers.
 *
 * Conventions
 *   * The graph is the user's in-CSR: indptr[N+1], indices[E] (source ids).  Edge e is the e-th
 *     entry of `indices`; dst(e) is the row that contains e; src(e) = indices[e].  User edge id ==
 *     position (SURVEY.md §8(c) reading #16, "separate array for edge ids").
 *   * All floating-point inputs and outputs are double; every sum is a plain loop in edge-id order
 *     with a double accumulator.  Row-major dense arrays, no padding.
 *   * `rows`/`nrows`: optional list of vertex ids to evaluate (NULL => all vertices in id order),
 *     so large graphs can be checked on sampled outputs one by one.
 *
 * Each function cites the passage it follows.  Readings of silent/garbled points are the ones
 * listed in DESIGN.md §3.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>
#ifdef _OPENMP
#include <omp.h>
#endif

enum { ORC_ACT_NONE = 0, ORC_ACT_RELU = 1, ORC_ACT_ELU = 2, ORC_ACT_SIGMOID = 3 };

/* ------------------------------------------------------------------------------------------ */
/* small helpers                                                                               */
/* ------------------------------------------------------------------------------------------ */

static int64_t* dst_of_edges(int64_t N, int64_t E, const int64_t* indptr) {
    int64_t* dst = (int64_t*)malloc(sizeof(int64_t) * (size_t)(E > 0 ? E : 1));
    for (int64_t v = 0; v < N; ++v)
        for (int64_t e = indptr[v]; e < indptr[v + 1]; ++e) dst[e] = v;
    return dst;
}

/* out-adjacency: out_ptr[N+1], out_eid[E] listing out-edges of each source in edge-id order */
static void out_adjacency(int64_t N, int64_t E, const int64_t* indices, int64_t** out_ptr, int64_t** out_eid) {
    int64_t* ptr = (int64_t*)calloc((size_t)(N + 1), sizeof(int64_t));
    int64_t* eid = (int64_t*)malloc(sizeof(int64_t) * (size_t)(E > 0 ? E : 1));
    for (int64_t e = 0; e < E; ++e) ptr[indices[e] + 1]++;
    for (int64_t u = 0; u < N; ++u) ptr[u + 1] += ptr[u];
    int64_t* fill = (int64_t*)malloc(sizeof(int64_t) * (size_t)(N + 1));
    memcpy(fill, ptr, sizeof(int64_t) * (size_t)(N + 1));
    for (int64_t e = 0; e < E; ++e) eid[fill[indices[e]]++] = e;   /* ascending e */
    free(fill);
    *out_ptr = ptr;
    *out_eid = eid;
}

static inline double act_fwd(int act, double x) {
    switch (act) {
        case ORC_ACT_RELU: return x > 0.0 ? x : 0.0;
        case ORC_ACT_ELU: return x > 0.0 ? x : expm1(x);
        case ORC_ACT_SIGMOID: return 1.0 / (1.0 + exp(-x));
        default: return x;
    }
}

/* derivative of the activation at the pre-activation value x */
static inline double act_grad(int act, double x) {
    switch (act) {
        case ORC_ACT_RELU: return x > 0.0 ? 1.0 : 0.0;
        case ORC_ACT_ELU: return x > 0.0 ? 1.0 : exp(x);
        case ORC_ACT_SIGMOID: { double s = 1.0 / (1.0 + exp(-x)); return s * (1.0 - s); }
        default: return 1.0;
    }
}

void orc_act_fwd(int act, int64_t n, const double* Z, double* Y) {
    for (int64_t i = 0; i < n; ++i) Y[i] = act_fwd(act, Z[i]);
}

void orc_act_bwd(int act, int64_t n, const double* Z, const double* dY, double* dZ) {
    for (int64_t i = 0; i < n; ++i) dZ[i] = dY[i] * act_grad(act, Z[i]);
}

/* ------------------------------------------------------------------------------------------ */
/* a1-a3: graph representation (§6.1, Fig. 7, §6.3.4,        */
/*        §6.3.5)                                                                    */
/* ------------------------------------------------------------------------------------------ */

typedef struct { int64_t key; int64_t id; } kv_t;                 /* vertex sort record */
typedef struct { int64_t a; int64_t b; int64_t e; } edge_key_t;   /* (primary, type, eid) */

static int cmp_kv(const void* x, const void* y) {
    const kv_t* p = (const kv_t*)x; const kv_t* q = (const kv_t*)y;
    if (p->key != q->key) return p->key < q->key ? -1 : 1;
    return p->id < q->id ? -1 : (p->id > q->id);
}
static int cmp_ek(const void* x, const void* y) {
    const edge_key_t* p = (const edge_key_t*)x; const edge_key_t* q = (const edge_key_t*)y;
    if (p->a != q->a) return p->a < q->a ? -1 : 1;
    if (p->b != q->b) return p->b < q->b ? -1 : 1;
    return p->e < q->e ? -1 : (p->e > q->e);
}

/*
 * Forward CSR, reverse CSR and edge-position map for the owned vertex range [row_begin,row_end).
 *
 *   fwd_perm  : owned vertices sorted by (in-degree desc, id asc)          -- L301, Fig. 7
 *   fwd row k : in-edges of fwd_perm[k] sorted by (type asc, eid asc)     -- Fig. 7
 *   rev_perm  : owned vertices sorted by (out-degree desc, id asc)         -- L301, L461
 *   rev row k : out-edges of rev_perm[k] sorted by (type asc, eid asc)    -- L461-L463, L475
 *   rev_pos[i]: position of edge rev_eid[i] in the "local-source forward" order: for the full range
 *               this is the forward CSR itself; for a partial range it is the list of edges whose
 *               source is owned, sorted by (dst id, type, eid) (SURVEY.md §8(e) LSF).
 * etypes may be NULL (then every type is 0).  Output arrays are caller-allocated:
 *   fwd_perm/rev_perm[n_loc], fwd_off/rev_off[n_loc+1], fwd_*[E_fwd], rev_*[E_rev],
 *   lsf_off[N+1] and lsf_eid[E_rev] (only written for a partial range; may be NULL otherwise).
 */
int orc_preprocess(int64_t N, int64_t E, const int64_t* indptr, const int64_t* indices,
                   const int32_t* etypes, int64_t row_begin, int64_t row_end,
                   int64_t* fwd_perm, int64_t* fwd_off, int64_t* fwd_src, int64_t* fwd_eid, int64_t* fwd_type,
                   int64_t* rev_perm, int64_t* rev_off, int64_t* rev_dst, int64_t* rev_eid, int64_t* rev_pos,
                   int64_t* rev_type, int64_t* lsf_off, int64_t* lsf_eid) {
    int64_t n_loc = row_end - row_begin;
    int64_t* dst = dst_of_edges(N, E, indptr);
    int64_t* outdeg = (int64_t*)calloc((size_t)(N > 0 ? N : 1), sizeof(int64_t));
    for (int64_t e = 0; e < E; ++e) outdeg[indices[e]]++;

    /* forward: sort owned vertices by (-indeg, id) */
    kv_t* kv = (kv_t*)malloc(sizeof(kv_t) * (size_t)(n_loc > 0 ? n_loc : 1));
    for (int64_t i = 0; i < n_loc; ++i) {
        int64_t v = row_begin + i;
        kv[i].key = -(indptr[v + 1] - indptr[v]);
        kv[i].id = v;
    }
    qsort(kv, (size_t)n_loc, sizeof(kv_t), cmp_kv);
    fwd_off[0] = 0;
    int64_t maxdeg = 0;
    for (int64_t k = 0; k < n_loc; ++k) {
        int64_t v = kv[k].id;
        fwd_perm[k] = v;
        int64_t b = indptr[v], d = indptr[v + 1] - indptr[v];
        if (d > maxdeg) maxdeg = d;
        edge_key_t* row = (edge_key_t*)malloc(sizeof(edge_key_t) * (size_t)(d > 0 ? d : 1));
        for (int64_t j = 0; j < d; ++j) {
            row[j].a = 0;
            row[j].b = etypes ? etypes[b + j] : 0;
            row[j].e = b + j;
        }
        qsort(row, (size_t)d, sizeof(edge_key_t), cmp_ek);
        for (int64_t j = 0; j < d; ++j) {
            int64_t p = fwd_off[k] + j;
            fwd_eid[p] = row[j].e;
            fwd_src[p] = indices[row[j].e];
            fwd_type[p] = row[j].b;
        }
        fwd_off[k + 1] = fwd_off[k] + d;
        free(row);
    }

    /* reverse: sort owned vertices by (-outdeg, id) */
    for (int64_t i = 0; i < n_loc; ++i) {
        int64_t u = row_begin + i;
        kv[i].key = -outdeg[u];
        kv[i].id = u;
    }
    qsort(kv, (size_t)n_loc, sizeof(kv_t), cmp_kv);
    int64_t *optr, *oeid;
    out_adjacency(N, E, indices, &optr, &oeid);
    rev_off[0] = 0;
    for (int64_t k = 0; k < n_loc; ++k) {
        int64_t u = kv[k].id;
        rev_perm[k] = u;
        int64_t d = optr[u + 1] - optr[u];
        edge_key_t* row = (edge_key_t*)malloc(sizeof(edge_key_t) * (size_t)(d > 0 ? d : 1));
        for (int64_t j = 0; j < d; ++j) {
            int64_t e = oeid[optr[u] + j];
            row[j].a = 0;
            row[j].b = etypes ? etypes[e] : 0;
            row[j].e = e;
        }
        qsort(row, (size_t)d, sizeof(edge_key_t), cmp_ek);
        for (int64_t j = 0; j < d; ++j) {
            int64_t p = rev_off[k] + j;
            rev_eid[p] = row[j].e;
            rev_dst[p] = dst[row[j].e];
            rev_type[p] = row[j].b;
        }
        rev_off[k + 1] = rev_off[k] + d;
        free(row);
    }
    int64_t E_rev = rev_off[n_loc];

    /* position map for rev_pos */
    int64_t* pos_of = (int64_t*)malloc(sizeof(int64_t) * (size_t)(E > 0 ? E : 1));
    for (int64_t e = 0; e < E; ++e) pos_of[e] = -1;
    if (row_begin == 0 && row_end == N) {
        for (int64_t p = 0; p < fwd_off[n_loc]; ++p) pos_of[fwd_eid[p]] = p;
    } else {
        edge_key_t* lsf = (edge_key_t*)malloc(sizeof(edge_key_t) * (size_t)(E_rev > 0 ? E_rev : 1));
        int64_t m = 0;
        for (int64_t e = 0; e < E; ++e) {
            if (indices[e] >= row_begin && indices[e] < row_end) {
                lsf[m].a = dst[e];
                lsf[m].b = etypes ? etypes[e] : 0;
                lsf[m].e = e;
                ++m;
            }
        }
        qsort(lsf, (size_t)m, sizeof(edge_key_t), cmp_ek);
        for (int64_t v = 0; v <= N; ++v) lsf_off[v] = 0;
        for (int64_t p = 0; p < m; ++p) {
            pos_of[lsf[p].e] = p;
            lsf_eid[p] = lsf[p].e;
            lsf_off[lsf[p].a + 1]++;
        }
        for (int64_t v = 0; v < N; ++v) lsf_off[v + 1] += lsf_off[v];
        free(lsf);
    }
    for (int64_t i = 0; i < E_rev; ++i) rev_pos[i] = pos_of[rev_eid[i]];

    free(pos_of); free(optr); free(oeid); free(kv); free(outdeg); free(dst);
    (void)maxdeg;
    return 0;
}

/* deg^-1/2 with deg clamped to >= 1 (SURVEY.md §8(c) reading #1: DGL "both" normalisation) */
void orc_degree_norms(int64_t N, int64_t E, const int64_t* indptr, const int64_t* indices,
                      double* in_norm, double* out_norm) {
    int64_t* outdeg = (int64_t*)calloc((size_t)(N > 0 ? N : 1), sizeof(int64_t));
    for (int64_t e = 0; e < E; ++e) outdeg[indices[e]]++;
    for (int64_t v = 0; v < N; ++v) {
        int64_t di = indptr[v + 1] - indptr[v];
        in_norm[v] = 1.0 / sqrt((double)(di > 1 ? di : 1));
        out_norm[v] = 1.0 / sqrt((double)(outdeg[v] > 1 ? outdeg[v] : 1));
    }
    free(outdeg);
}

/* ------------------------------------------------------------------------------------------ */
/* a4 / a11: dense transform (S-type ops run unfused in the backend; Fig. 2      */
/* f = W h written row-major as T = X W, SURVEY.md reading #4)                                  */
/* ------------------------------------------------------------------------------------------ */

/* Y[M,Nout] = X[M,K] W[K,Nout] (+ bias[Nout]) */
void orc_linear_fwd(int64_t M, int64_t K, int64_t Nout, const double* X, const double* W,
                    const double* bias, double* Y) {
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < M; ++i)
        for (int64_t j = 0; j < Nout; ++j) {
            double acc = bias ? bias[j] : 0.0;
            for (int64_t k = 0; k < K; ++k) acc += X[i * K + k] * W[k * Nout + j];
            Y[i * Nout + j] = acc;
        }
}

/* dX = dY W^T, dW = X^T dY, db = sum_i dY[i]  (each output optional) */
void orc_linear_bwd(int64_t M, int64_t K, int64_t Nout, const double* X, const double* W,
                    const double* dY, double* dX, double* dW, double* db) {
    if (dX) {
        #pragma omp parallel for schedule(static)
        for (int64_t i = 0; i < M; ++i)
            for (int64_t k = 0; k < K; ++k) {
                double acc = 0.0;
                for (int64_t j = 0; j < Nout; ++j) acc += dY[i * Nout + j] * W[k * Nout + j];
                dX[i * K + k] = acc;
            }
    }
    if (dW) {
        #pragma omp parallel for schedule(static)
        for (int64_t k = 0; k < K; ++k)
            for (int64_t j = 0; j < Nout; ++j) {
                double acc = 0.0;
                for (int64_t i = 0; i < M; ++i) acc += X[i * K + k] * dY[i * Nout + j];
                dW[k * Nout + j] = acc;
            }
    }
    if (db) {
        for (int64_t j = 0; j < Nout; ++j) {
            double acc = 0.0;
            for (int64_t i = 0; i < M; ++i) acc += dY[i * Nout + j];
            db[j] = acc;
        }
    }
}

/* ------------------------------------------------------------------------------------------ */
/* a5 / a8: GCN aggregation (Fig. 1 L85-L93: h_v' = sigma(b + sum_{u in N(v)} 1/norm *  */
/* h_u W); Fig. 3 L159 src lines 1-7; the APPNP propagation of [38] reuses it)                  */
/* ------------------------------------------------------------------------------------------ */

/* out[r,:] = dst_norm[v] * sum_{e in in(v)} src_norm[src(e)] * H[src(e),:],  v = rows[r] */
/* edge_w (optional, NEXT-3 edge dropout, reading #27): [E] multiplier of each edge's message by user edge id */
void orc_gcn_aggregate(int64_t N, int64_t E, const int64_t* indptr, const int64_t* indices, int64_t F,
                       const double* H, const double* src_norm, const double* dst_norm,
                       const int64_t* rows, int64_t nrows, double* out, const double* edge_w) {
    (void)E;
    if (!rows) nrows = N;
    #pragma omp parallel for schedule(dynamic, 64)
    for (int64_t r = 0; r < nrows; ++r) {
        int64_t v = rows ? rows[r] : r;
        double* o = out + r * F;
        for (int64_t f = 0; f < F; ++f) o[f] = 0.0;
        for (int64_t e = indptr[v]; e < indptr[v + 1]; ++e) {
            int64_t u = indices[e];
            double w = src_norm ? src_norm[u] : 1.0;
            if (edge_w) w *= edge_w[e];
            for (int64_t f = 0; f < F; ++f) o[f] += w * H[u * F + f];
        }
        double d = dst_norm ? dst_norm[v] : 1.0;
        for (int64_t f = 0; f < F; ++f) o[f] *= d;
    }
}

/* adjoint of orc_gcn_aggregate (§6.3.4: the backward aggregates over out-edges):
 * out[r,:] = src_norm[u] * sum_{e in out(u)} dst_norm[dst(e)] * G[dst(e),:],  u = rows[r] */
/* The whole graph's destination-of-edge and out-adjacency arrays (dst[E], optr[N+1], oeid[E]) that the
 * transposed loops below walk.  They are a pure function of the graph, so a caller timing a bounded row
 * sample (bench.py's cpu_baseline) builds them once and passes them in; NULL => each
 * call builds its own, as before.  Restructuring only: the arithmetic of every loop is unchanged. */
void orc_out_adjacency(int64_t N, int64_t E, const int64_t* indptr, const int64_t* indices,
                       int64_t* dst_out, int64_t* optr_out, int64_t* oeid_out) {
    int64_t* dst = dst_of_edges(N, E, indptr);
    int64_t *optr, *oeid;
    out_adjacency(N, E, indices, &optr, &oeid);
    memcpy(dst_out, dst, sizeof(int64_t) * (size_t)E);
    memcpy(optr_out, optr, sizeof(int64_t) * (size_t)(N + 1));
    memcpy(oeid_out, oeid, sizeof(int64_t) * (size_t)E);
    free(dst); free(optr); free(oeid);
}

void orc_gcn_aggregate_T(int64_t N, int64_t E, const int64_t* indptr, const int64_t* indices, int64_t F,
                         const double* G, const double* src_norm, const double* dst_norm,
                         const int64_t* rows, int64_t nrows, double* out, const double* edge_w,
                         const int64_t* adj_dst, const int64_t* adj_ptr, const int64_t* adj_eid) {
    int64_t *dst, *optr, *oeid;
    const int own = !(adj_dst && adj_ptr && adj_eid);
    if (own) {
        dst = dst_of_edges(N, E, indptr);
        out_adjacency(N, E, indices, &optr, &oeid);
    } else {
        dst = (int64_t*)adj_dst; optr = (int64_t*)adj_ptr; oeid = (int64_t*)adj_eid;
    }
    if (!rows) nrows = N;
    #pragma omp parallel for schedule(dynamic, 64)
    for (int64_t r = 0; r < nrows; ++r) {
        int64_t u = rows ? rows[r] : r;
        double* o = out + r * F;
        for (int64_t f = 0; f < F; ++f) o[f] = 0.0;
        for (int64_t p = optr[u]; p < optr[u + 1]; ++p) {
            int64_t v = dst[oeid[p]];
            double w = dst_norm ? dst_norm[v] : 1.0;
            if (edge_w) w *= edge_w[oeid[p]];
            for (int64_t f = 0; f < F; ++f) o[f] += w * G[v * F + f];
        }
        double s = src_norm ? src_norm[u] : 1.0;
        for (int64_t f = 0; f < F; ++f) o[f] *= s;
    }
    if (own) { free(optr); free(oeid); free(dst); }
}

/* OpenMP thread count for the timed baselines (bench.py records single-threaded numbers too) */
void orc_set_num_threads(int n) {
#ifdef _OPENMP
    omp_set_num_threads(n);
#else
    (void)n;
#endif
}

/* ------------------------------------------------------------------------------------------ */
/* a6 / a9: GAT (Fig. 2 L95-L123, Fig. 3 L159 src lines 9-23 with the typos of         */
/* SURVEY.md reading #4 fixed; heads independent, reading #7; LeakyReLU slope, reading #6)      */
/* ------------------------------------------------------------------------------------------ */

/* el[u,h] = sum_f T[u,h,f] a_l[h,f];  er[v,h] = sum_f T[v,h,f] a_r[h,f]   (Fig. 2: e_u = f_u^T attn_u) */
void orc_gat_attn_proj(int64_t N, int64_t H, int64_t F, const double* T, const double* a_l,
                       const double* a_r, double* el, double* er) {
    for (int64_t u = 0; u < N; ++u)
        for (int64_t h = 0; h < H; ++h) {
            double sl = 0.0, sr = 0.0;
            for (int64_t f = 0; f < F; ++f) {
                sl += T[(u * H + h) * F + f] * a_l[h * F + f];
                sr += T[(u * H + h) * F + f] * a_r[h * F + f];
            }
            el[u * H + h] = sl;
            er[u * H + h] = sr;
        }
}

static inline double lrelu(double x, double slope) { return x > 0.0 ? x : slope * x; }

/*
 * Forward: for each v, h:  e_uv = LeakyReLU(el[u,h] + er[v,h]);
 *   a_uv = exp(e_uv) / sum_{u' in N(v)} exp(e_u'v)      (computed max-subtracted, reading #5)
 *   A[v,h,:] = sum_u a_uv T[u,h,:];  lse[v,h] = log sum exp(e_uv)  (-inf for an empty row)
 * alpha (optional): alpha[e*H + h] for every edge, by edge id.
 */
/* mask (optional, NEXT-3 attention dropout, reading #27): [E, H] multiplier of the attention weight of edge e
 * (user edge id) in the aggregation, A = sum_e a_e mask_e T_u (the softmax itself is not masked) */
void orc_gat_fwd(int64_t N, int64_t E, const int64_t* indptr, const int64_t* indices, int64_t H, int64_t F,
                 const double* T, const double* el, const double* er, double slope,
                 const int64_t* rows, int64_t nrows, double* A, double* lse, double* alpha, const double* mask) {
    (void)E;
    if (!rows) nrows = N;
    #pragma omp parallel for schedule(dynamic, 64)
    for (int64_t r = 0; r < nrows; ++r) {
        int64_t v = rows ? rows[r] : r;
        for (int64_t h = 0; h < H; ++h) {
            double* a = A + (r * H + h) * F;
            for (int64_t f = 0; f < F; ++f) a[f] = 0.0;
            if (indptr[v + 1] == indptr[v]) { lse[r * H + h] = -INFINITY; continue; }
            double m = -INFINITY;
            for (int64_t e = indptr[v]; e < indptr[v + 1]; ++e) {
                double z = lrelu(el[indices[e] * H + h] + er[v * H + h], slope);
                if (z > m) m = z;
            }
            double S = 0.0;
            for (int64_t e = indptr[v]; e < indptr[v + 1]; ++e)
                S += exp(lrelu(el[indices[e] * H + h] + er[v * H + h], slope) - m);
            for (int64_t e = indptr[v]; e < indptr[v + 1]; ++e) {
                int64_t u = indices[e];
                double al = exp(lrelu(el[u * H + h] + er[v * H + h], slope) - m) / S;
                if (alpha) alpha[e * H + h] = al;
                const double mk = mask ? mask[e * H + h] : 1.0;
                for (int64_t f = 0; f < F; ++f) a[f] += al * mk * T[(u * H + h) * F + f];
            }
            lse[r * H + h] = m + log(S);
        }
    }
}

/*
 * Backward of orc_gat_fwd w.r.t. T, el, er given dA = dL/dA (the plain way: explicit softmax
 * Jacobian per (v,h), dz_e = a_e (g_e - sum_e' a_e' g_e'), g_e = <dA[v,h], T[src,h]>;
 * ds_e = dz_e * LeakyReLU'(s_e) with LeakyReLU'(0) = slope).
 *   dT[u,h,:] = sum_{e in out(u)} a_e dA[dst,h,:]     del[u,h] = sum_{e in out(u)} ds_e
 *   der[v,h]  = sum_{e in in(v)} ds_e
 * Pass 1 (all v) computes per-(v,h) softmax statistics and der; pass 2 evaluates the source-side
 * sums for `rows` (NULL => all).  dT/del are [nrows,...]; der is [N,H].
 * With the optional attention-dropout mask of orc_gat_fwd, dA_e/d a_e = mask_e g_e: g_e is replaced by
 * mask_e g_e in the Jacobian and dT[u] gets a_e mask_e dA[dst].
 */
void orc_gat_bwd(int64_t N, int64_t E, const int64_t* indptr, const int64_t* indices, int64_t H, int64_t F,
                 const double* T, const double* el, const double* er, double slope, const double* dA,
                 const int64_t* rows, int64_t nrows, double* dT, double* del, double* der, const double* mask,
                 const int64_t* adj_dst, const int64_t* adj_ptr, const int64_t* adj_eid) {
    double* mx = (double*)malloc(sizeof(double) * (size_t)(N * H > 0 ? N * H : 1));
    double* sm = (double*)malloc(sizeof(double) * (size_t)(N * H > 0 ? N * H : 1));
    double* gb = (double*)malloc(sizeof(double) * (size_t)(N * H > 0 ? N * H : 1));
    #pragma omp parallel for schedule(dynamic, 64)
    for (int64_t v = 0; v < N; ++v) {
        for (int64_t h = 0; h < H; ++h) {
            double m = -INFINITY, S = 0.0, gbar = 0.0, dsum = 0.0;
            for (int64_t e = indptr[v]; e < indptr[v + 1]; ++e) {
                double z = lrelu(el[indices[e] * H + h] + er[v * H + h], slope);
                if (z > m) m = z;
            }
            for (int64_t e = indptr[v]; e < indptr[v + 1]; ++e)
                S += exp(lrelu(el[indices[e] * H + h] + er[v * H + h], slope) - m);
            for (int64_t e = indptr[v]; e < indptr[v + 1]; ++e) {
                int64_t u = indices[e];
                double al = exp(lrelu(el[u * H + h] + er[v * H + h], slope) - m) / S;
                double g = 0.0;
                for (int64_t f = 0; f < F; ++f) g += dA[(v * H + h) * F + f] * T[(u * H + h) * F + f];
                if (mask) g *= mask[e * H + h];
                gbar += al * g;
            }
            for (int64_t e = indptr[v]; e < indptr[v + 1]; ++e) {
                int64_t u = indices[e];
                double s = el[u * H + h] + er[v * H + h];
                double al = exp(lrelu(s, slope) - m) / S;
                double g = 0.0;
                for (int64_t f = 0; f < F; ++f) g += dA[(v * H + h) * F + f] * T[(u * H + h) * F + f];
                if (mask) g *= mask[e * H + h];
                dsum += al * (g - gbar) * (s > 0.0 ? 1.0 : slope);
            }
            mx[v * H + h] = m; sm[v * H + h] = S; gb[v * H + h] = gbar;
            der[v * H + h] = dsum;
        }
    }
    int64_t *dst, *optr, *oeid;          /* prebuilt adjacency (orc_out_adjacency) or built here */
    const int own = !(adj_dst && adj_ptr && adj_eid);
    if (own) {
        dst = dst_of_edges(N, E, indptr);
        out_adjacency(N, E, indices, &optr, &oeid);
    } else {
        dst = (int64_t*)adj_dst; optr = (int64_t*)adj_ptr; oeid = (int64_t*)adj_eid;
    }
    if (!rows) nrows = N;
    #pragma omp parallel for schedule(dynamic, 64)
    for (int64_t r = 0; r < nrows; ++r) {
        int64_t u = rows ? rows[r] : r;
        for (int64_t h = 0; h < H; ++h) {
            double* o = dT + (r * H + h) * F;
            for (int64_t f = 0; f < F; ++f) o[f] = 0.0;
            double dl = 0.0;
            for (int64_t p = optr[u]; p < optr[u + 1]; ++p) {
                int64_t v = dst[oeid[p]];
                double s = el[u * H + h] + er[v * H + h];
                double al = exp(lrelu(s, slope) - mx[v * H + h]) / sm[v * H + h];
                const double mk = mask ? mask[oeid[p] * H + h] : 1.0;
                double g = 0.0;
                for (int64_t f = 0; f < F; ++f) g += dA[(v * H + h) * F + f] * T[(u * H + h) * F + f];
                dl += al * (mk * g - gb[v * H + h]) * (s > 0.0 ? 1.0 : slope);
                for (int64_t f = 0; f < F; ++f) o[f] += al * mk * dA[(v * H + h) * F + f];
            }
            del[r * H + h] = dl;
        }
    }
    if (own) { free(optr); free(oeid); free(dst); }
    free(mx); free(sm); free(gb);
}

/* ------------------------------------------------------------------------------------------ */
/* a7 / a10: R-GCN (§6.3.5: sum over edges of a type, then over types;       */
/* layer formula of [53], SURVEY.md §8(c) R-GCN, reading #17)                                   */
/* ------------------------------------------------------------------------------------------ */

/* norm_by_eid[e] = 1 / |{e' in in(dst(e)) : type(e') = type(e)}|   (c_{v,r} of [53]) */
void orc_rgcn_norm(int64_t N, int64_t E, const int64_t* indptr, const int32_t* etypes, int32_t R,
                   double* norm_by_eid) {
    (void)E;
    int64_t* cnt = (int64_t*)calloc((size_t)(R > 0 ? R : 1), sizeof(int64_t));
    for (int64_t v = 0; v < N; ++v) {
        for (int64_t e = indptr[v]; e < indptr[v + 1]; ++e) cnt[etypes[e]]++;
        for (int64_t e = indptr[v]; e < indptr[v + 1]; ++e) norm_by_eid[e] = 1.0 / (double)cnt[etypes[e]];
        for (int64_t e = indptr[v]; e < indptr[v + 1]; ++e) cnt[etypes[e]] = 0;
    }
    free(cnt);
}

/* out[r,:] = sum_{e in in(v)} norm[e] * X[src(e),:] W[type(e)]     (W is [R, Fin, Fout]) */
void orc_rgcn_fwd(int64_t N, int64_t E, const int64_t* indptr, const int64_t* indices, const int32_t* etypes,
                  int64_t Fin, int64_t Fout, const double* X, const double* W, const double* norm,
                  const int64_t* rows, int64_t nrows, double* out) {
    (void)E;
    if (!rows) nrows = N;
    #pragma omp parallel for schedule(dynamic, 64)
    for (int64_t r = 0; r < nrows; ++r) {
        int64_t v = rows ? rows[r] : r;
        double* o = out + r * Fout;
        for (int64_t j = 0; j < Fout; ++j) o[j] = 0.0;
        for (int64_t e = indptr[v]; e < indptr[v + 1]; ++e) {
            int64_t u = indices[e];
            const double* Wr = W + (int64_t)etypes[e] * Fin * Fout;
            for (int64_t j = 0; j < Fout; ++j) {
                double t = 0.0;
                for (int64_t i = 0; i < Fin; ++i) t += X[u * Fin + i] * Wr[i * Fout + j];
                o[j] += norm[e] * t;
            }
        }
    }
}

/* dX[u,:] = sum_{e in out(u)} norm[e] dA[dst(e),:] W[type(e)]^T ;
 * dW[r]   = sum_{e : type(e) = r} norm[e] X[src(e),:]^T dA[dst(e),:]      (both optional) */
void orc_rgcn_bwd(int64_t N, int64_t E, const int64_t* indptr, const int64_t* indices, const int32_t* etypes,
                  int32_t R, int64_t Fin, int64_t Fout, const double* X, const double* W, const double* norm,
                  const double* dA, double* dX, double* dW) {
    int64_t* dst = dst_of_edges(N, E, indptr);
    if (dX) {
        int64_t *optr, *oeid;
        out_adjacency(N, E, indices, &optr, &oeid);
        #pragma omp parallel for schedule(dynamic, 64)
        for (int64_t u = 0; u < N; ++u) {
            double* o = dX + u * Fin;
            for (int64_t i = 0; i < Fin; ++i) o[i] = 0.0;
            for (int64_t p = optr[u]; p < optr[u + 1]; ++p) {
                int64_t e = oeid[p], v = dst[e];
                const double* Wr = W + (int64_t)etypes[e] * Fin * Fout;
                for (int64_t i = 0; i < Fin; ++i) {
                    double t = 0.0;
                    for (int64_t j = 0; j < Fout; ++j) t += dA[v * Fout + j] * Wr[i * Fout + j];
                    o[i] += norm[e] * t;
                }
            }
        }
        free(optr); free(oeid);
    }
    if (dW) {
        #pragma omp parallel for schedule(dynamic, 1)
        for (int32_t r = 0; r < R; ++r) {
            double* o = dW + (int64_t)r * Fin * Fout;
            for (int64_t k = 0; k < Fin * Fout; ++k) o[k] = 0.0;
            for (int64_t e = 0; e < E; ++e) {
                if (etypes[e] != r) continue;
                int64_t u = indices[e], v = dst[e];
                for (int64_t i = 0; i < Fin; ++i)
                    for (int64_t j = 0; j < Fout; ++j) o[i * Fout + j] += norm[e] * X[u * Fin + i] * dA[v * Fout + j];
            }
        }
    }
    free(dst);
}

/* ------------------------------------------------------------------------------------------ */
/* NEXT-2: R-GCN as the paper ran it (Table 2/3 L485, L1219-L1227: aifb / mutag / bgs with a     */
/* featureless input layer).  Layer of [53] with basis decomposition (reading #27):              */
/*   W_r = sum_b a[r,b] V_b ; featureless input h_u = one-hot(u) => h_u W_r = W_r[u,:]            */
/* V is stored [N, B, F] (V[u,b,:] = row u of basis b), a is [R, B].                             */
/* ------------------------------------------------------------------------------------------ */

/* out[r,:] = sum_{e in in(v)} norm[e] * W_{type(e)}[src(e),:],  W_t[u,:] = sum_b a[t,b] V[u,b,:] */
void orc_rgcn_basis_fwd(int64_t N, int64_t E, const int64_t* indptr, const int64_t* indices,
                        const int32_t* etypes, int64_t B, int64_t F, const double* V, const double* a,
                        const double* norm, const int64_t* rows, int64_t nrows, double* out) {
    (void)E;
    if (!rows) nrows = N;
    #pragma omp parallel for schedule(dynamic, 64)
    for (int64_t r = 0; r < nrows; ++r) {
        int64_t v = rows ? rows[r] : r;
        double* o = out + r * F;
        for (int64_t f = 0; f < F; ++f) o[f] = 0.0;
        for (int64_t e = indptr[v]; e < indptr[v + 1]; ++e) {
            int64_t u = indices[e], t = etypes[e];
            for (int64_t f = 0; f < F; ++f) {
                double w = 0.0;                               /* W_t[u,f] */
                for (int64_t b = 0; b < B; ++b) w += a[t * B + b] * V[(u * B + b) * F + f];
                o[f] += norm[e] * w;
            }
        }
    }
}

/* VJP of orc_rgcn_basis_fwd given dA = dL/d out (all N rows):
 *   dV[u,b,:] = sum_{e in out(u)} norm[e] a[type(e),b] dA[dst(e),:]
 *   da[t,b]   = sum_{e : type(e) = t} norm[e] <V[src(e),b,:], dA[dst(e),:]>      (both optional) */
void orc_rgcn_basis_bwd(int64_t N, int64_t E, const int64_t* indptr, const int64_t* indices,
                        const int32_t* etypes, int32_t R, int64_t B, int64_t F, const double* V,
                        const double* a, const double* norm, const double* dA, double* dV, double* da) {
    int64_t* dst = dst_of_edges(N, E, indptr);
    if (dV) {
        int64_t *optr, *oeid;
        out_adjacency(N, E, indices, &optr, &oeid);
        #pragma omp parallel for schedule(dynamic, 64)
        for (int64_t u = 0; u < N; ++u) {
            double* o = dV + u * B * F;
            for (int64_t k = 0; k < B * F; ++k) o[k] = 0.0;
            for (int64_t p = optr[u]; p < optr[u + 1]; ++p) {
                int64_t e = oeid[p], v = dst[e], t = etypes[e];
                for (int64_t b = 0; b < B; ++b)
                    for (int64_t f = 0; f < F; ++f) o[b * F + f] += norm[e] * a[t * B + b] * dA[v * F + f];
            }
        }
        free(optr); free(oeid);
    }
    if (da) {
        #pragma omp parallel for schedule(dynamic, 1)
        for (int32_t t = 0; t < R; ++t) {
            for (int64_t b = 0; b < B; ++b) da[(int64_t)t * B + b] = 0.0;
            for (int64_t e = 0; e < E; ++e) {
                if (etypes[e] != t) continue;
                int64_t u = indices[e], v = dst[e];
                for (int64_t b = 0; b < B; ++b) {
                    double d = 0.0;
                    for (int64_t f = 0; f < F; ++f) d += V[(u * B + b) * F + f] * dA[v * F + f];
                    da[(int64_t)t * B + b] += norm[e] * d;
                }
            }
        }
    }
    free(dst);
}

/* ------------------------------------------------------------------------------------------ */
/* NEXT-3: reproducible dropout ("further processed using a Dropout layer"; DGL    */
/* default configs, L481).  Counter-based mask, reading #27:                          */
/*   key   = sm64(seed ^ sm64((site << 32) | step))                                             */
/*   keep(i) <=> (sm64(key ^ i) >> 40) >= thr,  thr = round(p * 2^24)                            */
/* with sm64 = Vigna's splitmix64 output function; i = global element index row * F + col.      */
/* ------------------------------------------------------------------------------------------ */
static uint64_t sm64(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

uint64_t orc_sm64(uint64_t z) { return sm64(z); }

/* mask[i] = keep(idx0 + i) ? 1 : 0 for i < n; p is the fp32 drop probability */
void orc_dropout_keep(uint64_t seed, uint32_t site, int32_t step, int64_t idx0, int64_t n, float p, uint8_t* mask) {
    const uint64_t key = sm64(seed ^ sm64(((uint64_t)site << 32) | (uint32_t)step));
    const uint32_t thr = (uint32_t)llround((double)p * 16777216.0);
    for (int64_t i = 0; i < n; ++i) mask[i] = (uint8_t)((sm64(key ^ (uint64_t)(idx0 + i)) >> 40) >= thr);
}

/* ------------------------------------------------------------------------------------------ */
/* training-step pieces around the hot path (DGL default training loop)         */
/* ------------------------------------------------------------------------------------------ */

/* mean softmax cross-entropy over M rows; dlogits = (softmax - onehot) / M */
double orc_softmax_xent(int64_t M, int64_t C, const double* logits, const int64_t* labels, double* dlogits) {
    double loss = 0.0;
    for (int64_t i = 0; i < M; ++i) {
        const double* z = logits + i * C;
        double m = -INFINITY;
        for (int64_t c = 0; c < C; ++c) if (z[c] > m) m = z[c];
        double S = 0.0;
        for (int64_t c = 0; c < C; ++c) S += exp(z[c] - m);
        double lse = m + log(S);
        loss += lse - z[labels[i]];
        if (dlogits)
            for (int64_t c = 0; c < C; ++c)
                dlogits[i * C + c] = (exp(z[c] - lse) - (c == labels[i] ? 1.0 : 0.0)) / (double)M;
    }
    return loss / (double)M;
}

/* one Adam step (Kingma & Ba, Alg. 1) at step t >= 1, in place */
void orc_adam(int64_t n, double* param, const double* grad, double* m, double* v, double lr, double b1,
              double b2, double eps, int64_t t) {
    double c1 = 1.0 - pow(b1, (double)t), c2 = 1.0 - pow(b2, (double)t);
    for (int64_t i = 0; i < n; ++i) {
        m[i] = b1 * m[i] + (1.0 - b1) * grad[i];
        v[i] = b2 * v[i] + (1.0 - b2) * grad[i] * grad[i];
        double mh = m[i] / c1, vh = v[i] / c2;
        param[i] -= lr * mh / (sqrt(vh) + eps);
    }
}
