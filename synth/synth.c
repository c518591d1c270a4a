/*
 * synth.c -- seeded synthetic-input generator shared by the CPU oracle tests and the GPU path.
 *
 * This module holds NO arithmetic of the Seastar method (no aggregation, no softmax, no
 * normalisation, no sorting by degree).  It only draws graphs and tensors whose *shapes* follow
 * the paper's datasets (Table 2) and the recipe in SURVEY.md §8(d):
 *
 *   * counter-based RNG   u(seed, i) = splitmix64(seed ^ (i * 0x9E3779B97F4A7C15)), top 53 bits;
 *   * Chung-Lu power-law graphs: vertex rank r has weight (r+1)^-s; ranks are mapped to vertex ids
 *     by a seeded Fisher-Yates shuffle so hubs are scattered over the id space;
 *   * symmetric graphs emit each drawn pair (a,b), a != b, in both directions, then optionally one
 *     self-loop per vertex (DGL example convention);
 *   * directed typed graphs (AM-shaped R-GCN input) draw dst ~ w_in, src ~ w_out and an edge type
 *     from a Zipf(R, a) law;
 *   * the user CSR is produced by a counting sort on dst that is stable in generation order, so
 *     user edge id e == position in `indices` (SURVEY.md §8(c) reading #16).
 *
 * Every draw is a pure function of (seed, counter), so the output is independent of the number
 * of OpenMP threads.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>

#define GOLDEN 0x9E3779B97F4A7C15ULL
#define RETRY  0xD1B54A32D192ED03ULL

static inline uint64_t splitmix64(uint64_t z) {
    z += GOLDEN;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}
static inline uint64_t ctr(uint64_t seed, uint64_t i) { return splitmix64(seed ^ (i * GOLDEN)); }
static inline double u01(uint64_t seed, uint64_t i) { return (double)(ctr(seed, i) >> 11) * 0x1.0p-53; }

uint64_t synth_u64(uint64_t seed, uint64_t i) { return ctr(seed, i); }
double synth_u01(uint64_t seed, uint64_t i) { return u01(seed, i); }

/* rank -> vertex id permutation (Fisher-Yates driven by the counter RNG) */
static void shuffle_ids(int64_t n, uint64_t seed, int32_t* perm) {
    for (int64_t i = 0; i < n; ++i) perm[i] = (int32_t)i;
    for (int64_t i = n - 1; i > 0; --i) {
        int64_t j = (int64_t)(u01(seed, (uint64_t)i) * (double)(i + 1));
        if (j > i) j = i;
        int32_t t = perm[i]; perm[i] = perm[j]; perm[j] = t;
    }
}

/* cumulative weights of (r+1)^-s, r = 0..n-1 */
static double* powerlaw_cdf(int64_t n, double s) {
    double* cdf = (double*)malloc(sizeof(double) * (size_t)n);
    double acc = 0.0;
    for (int64_t r = 0; r < n; ++r) { acc += pow((double)(r + 1), -s); cdf[r] = acc; }
    return cdf;
}

/* smallest r with cdf[r] > u * cdf[n-1] */
static inline int64_t draw(const double* cdf, int64_t n, double u) {
    double x = u * cdf[n - 1];
    int64_t lo = 0, hi = n - 1;
    while (lo < hi) {
        int64_t mid = lo + ((hi - lo) >> 1);
        if (cdf[mid] > x) hi = mid; else lo = mid + 1;
    }
    return lo;
}

/* stable counting sort of (src,dst[,type]) by dst -> user CSR */
static void to_csr(int64_t N, int64_t E, const int32_t* src, const int32_t* dst, const int32_t* typ,
                   int64_t* indptr, int64_t* indices, int32_t* etypes) {
    memset(indptr, 0, sizeof(int64_t) * (size_t)(N + 1));
    for (int64_t e = 0; e < E; ++e) indptr[dst[e] + 1]++;
    for (int64_t v = 0; v < N; ++v) indptr[v + 1] += indptr[v];
    int64_t* fill = (int64_t*)malloc(sizeof(int64_t) * (size_t)N);
    memcpy(fill, indptr, sizeof(int64_t) * (size_t)N);
    for (int64_t e = 0; e < E; ++e) {
        int64_t p = fill[dst[e]]++;
        indices[p] = src[e];
        if (etypes) etypes[p] = typ[e];
    }
    free(fill);
}

/*
 * Symmetric power-law graph.  E_dir directed non-loop edges (E_dir/2 pairs in both directions,
 * plus one extra directed edge when E_dir is odd) and, if self_loops, N self-loops.
 * Output: indptr[N+1], indices[E_dir + (self_loops ? N : 0)].
 */
int synth_powerlaw_sym(int64_t N, int64_t E_dir, double s, uint64_t seed, int self_loops,
                       int64_t* indptr, int64_t* indices) {
    if (N < 2) return 1;
    int64_t E = E_dir + (self_loops ? N : 0);
    int32_t* perm = (int32_t*)malloc(sizeof(int32_t) * (size_t)N);
    shuffle_ids(N, seed + 1, perm);
    double* cdf = powerlaw_cdf(N, s);
    int32_t* src = (int32_t*)malloc(sizeof(int32_t) * (size_t)E);
    int32_t* dst = (int32_t*)malloc(sizeof(int32_t) * (size_t)E);
    int64_t P = E_dir / 2, extra = E_dir % 2;
    #pragma omp parallel for schedule(static)
    for (int64_t k = 0; k < P + extra; ++k) {
        int32_t a, b;
        for (uint64_t t = 0;; ++t) {
            uint64_t sd = seed + t * RETRY;
            a = perm[draw(cdf, N, u01(sd, 2 * (uint64_t)k))];
            b = perm[draw(cdf, N, u01(sd, 2 * (uint64_t)k + 1))];
            if (a != b) break;
        }
        src[2 * k] = a; dst[2 * k] = b;
        if (k < P) { src[2 * k + 1] = b; dst[2 * k + 1] = a; }
    }
    if (self_loops)
        for (int64_t v = 0; v < N; ++v) { src[E_dir + v] = (int32_t)v; dst[E_dir + v] = (int32_t)v; }
    to_csr(N, E, src, dst, NULL, indptr, indices, NULL);
    free(src); free(dst); free(cdf); free(perm);
    return 0;
}

/*
 * Directed typed power-law graph (AM-shaped).  E edges, no self-loops, no symmetrisation.
 * dst ~ (r+1)^-s_in, src ~ (r+1)^-s_out (independent shuffles), type ~ Zipf(R, zipf_a).
 */
int synth_powerlaw_directed_typed(int64_t N, int64_t E, double s_in, double s_out, int32_t R,
                                  double zipf_a, uint64_t seed,
                                  int64_t* indptr, int64_t* indices, int32_t* etypes) {
    if (N < 2 || R < 1) return 1;
    int32_t* perm_in = (int32_t*)malloc(sizeof(int32_t) * (size_t)N);
    int32_t* perm_out = (int32_t*)malloc(sizeof(int32_t) * (size_t)N);
    shuffle_ids(N, seed + 1, perm_in);
    shuffle_ids(N, seed + 2, perm_out);
    double* cdf_in = powerlaw_cdf(N, s_in);
    double* cdf_out = powerlaw_cdf(N, s_out);
    double* cdf_t = powerlaw_cdf(R, zipf_a);
    int32_t* src = (int32_t*)malloc(sizeof(int32_t) * (size_t)E);
    int32_t* dst = (int32_t*)malloc(sizeof(int32_t) * (size_t)E);
    int32_t* typ = (int32_t*)malloc(sizeof(int32_t) * (size_t)E);
    #pragma omp parallel for schedule(static)
    for (int64_t k = 0; k < E; ++k) {
        int32_t a, b;
        uint64_t sd = seed;
        for (uint64_t t = 0;; ++t) {
            sd = seed + t * RETRY;
            b = perm_in[draw(cdf_in, N, u01(sd, 3 * (uint64_t)k))];
            a = perm_out[draw(cdf_out, N, u01(sd, 3 * (uint64_t)k + 1))];
            if (a != b) break;
        }
        src[k] = a; dst[k] = b;
        typ[k] = (int32_t)draw(cdf_t, R, u01(sd, 3 * (uint64_t)k + 2));
    }
    to_csr(N, E, src, dst, typ, indptr, indices, etypes);
    free(src); free(dst); free(typ); free(cdf_in); free(cdf_out); free(cdf_t);
    free(perm_in); free(perm_out);
    return 0;
}

/* out[i] = lo + (hi - lo) * u(seed, i), rounded to fp32 */
void synth_uniform_f32(uint64_t seed, int64_t n, double lo, double hi, float* out) {
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) out[i] = (float)(lo + (hi - lo) * u01(seed, (uint64_t)i));
}

/* out[i] = floor(C * u(seed, i)) in [0, C) */
void synth_labels(uint64_t seed, int64_t n, int32_t C, int64_t* out) {
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) {
        int64_t c = (int64_t)(u01(seed, (uint64_t)i) * (double)C);
        out[i] = c >= C ? C - 1 : c;
    }
}
