/*
 * datagen/gen.c -- seeded synthetic workload generators.
 *
 * This module is shared by BOTH sides of the parity check (oracle/ and the
 * CUDA path); it therefore holds NONE of the method's arithmetic: no window
 * condensation, no SpMM.  It only produces canonical CSR sparsity patterns and
 * value arrays from a counter-based generator, so the output is a pure
 * function of (seed, row/element index) and independent of the OpenMP thread
 * count.
 *
 * Generators
 *   G1  locality power-law graph (Cora/arxiv/reddit/products-shaped inputs):
 *       Pareto row degrees, each column drawn with prob p_local from the row's
 *       aligned community block of S columns, else from a Zipf(beta) popularity
 *       law over a seeded permutation of the column ids.  Shapes follow the
 *       paper's Table 1 and Table 2's MeanNnzTC targets
 *       (PAPER.md:133-146), used as calibration targets only.
 *   G2  banded/FEM matrix with long-row outliers (SuiteSparse-shaped).
 *
 * Randomness: rng(seed, stream, ctr) = splitmix64-style mixing of a
 * (seed, stream, counter) triple.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>

static inline uint64_t mix64(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}
static inline uint64_t rng(uint64_t seed, uint64_t stream, uint64_t ctr) {
    return mix64(mix64(seed * 0xD1B54A32D192ED03ull ^ (stream + 0x632BE59BD9B4E019ull)) + ctr);
}
static inline double u01(uint64_t x) { return (double)(x >> 11) * (1.0 / 9007199254740992.0); }

enum { ST_DEG = 1, ST_RND = 2, ST_COL = 3, ST_PERM = 4, ST_OUT = 5 };

/* ---------------------------------------------------------------- helpers */
static int cmp_i32(const void* a, const void* b) {
    int32_t x = *(const int32_t*)a, y = *(const int32_t*)b;
    return (x > y) - (x < y);
}
/* sort + unique in place, returns new length */
static int64_t sort_unique(int32_t* v, int64_t n) {
    if (n <= 1) return n;
    qsort(v, (size_t)n, sizeof(int32_t), cmp_i32);
    int64_t m = 1;
    for (int64_t i = 1; i < n; ++i)
        if (v[i] != v[m - 1]) v[m++] = v[i];
    return m;
}

/* ------------------------------------------------------------- G1 degrees */
static int64_t deg_of(double w, double r, double s, int64_t dmax) {
    double d = floor(w * s + r);
    if (d < 1) d = 1;
    if (d > (double)dmax) d = (double)dmax;
    return (int64_t)d;
}

/* Pareto(alpha) row weights, stochastic rounding, scale s bisected so that
 * sum(deg) is as close as possible to nnz_target.  deg_i in [1, d_max]. */
int64_t dg_powerlaw_degrees(int64_t M, int64_t nnz_target, double alpha, int64_t d_max,
                            uint64_t seed, int32_t* deg) {
    if (M <= 0) return 0;
    double* w = (double*)malloc(sizeof(double) * (size_t)M);
    double* r = (double*)malloc(sizeof(double) * (size_t)M);
    if (!w || !r) { free(w); free(r); return -1; }
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < M; ++i) {
        double u = u01(rng(seed, ST_DEG, (uint64_t)i));
        if (u < 1e-300) u = 1e-300;
        w[i] = pow(u, -1.0 / (alpha - 1.0));
        r[i] = u01(rng(seed, ST_RND, (uint64_t)i));
    }
    double lo = 0.0, hi = 1.0;
    for (;;) {  /* grow hi until the sum reaches the target (or saturates) */
        int64_t s = 0;
        #pragma omp parallel for reduction(+ : s) schedule(static)
        for (int64_t i = 0; i < M; ++i) s += deg_of(w[i], r[i], hi, d_max);
        if (s >= nnz_target || hi > 1e12) break;
        hi *= 2.0;
    }
    for (int it = 0; it < 100; ++it) {
        double mid = 0.5 * (lo + hi);
        int64_t s = 0;
        #pragma omp parallel for reduction(+ : s) schedule(static)
        for (int64_t i = 0; i < M; ++i) s += deg_of(w[i], r[i], mid, d_max);
        if (s < nnz_target) lo = mid; else hi = mid;
    }
    int64_t total = 0;
    #pragma omp parallel for reduction(+ : total) schedule(static)
    for (int64_t i = 0; i < M; ++i) { deg[i] = (int32_t)deg_of(w[i], r[i], hi, d_max); total += deg[i]; }
    free(w); free(r);
    return total;
}

/* Zipf(beta) CDF over ranks 1..K (double[K]) and a seeded permutation of 0..K-1. */
int dg_zipf_table(int64_t K, double beta, uint64_t seed, double* cdf, int32_t* perm) {
    double acc = 0.0;
    for (int64_t q = 0; q < K; ++q) { acc += pow((double)(q + 1), -beta); cdf[q] = acc; }
    for (int64_t q = 0; q < K; ++q) cdf[q] /= acc;
    cdf[K - 1] = 1.0;
    for (int64_t q = 0; q < K; ++q) perm[q] = (int32_t)q;
    for (int64_t q = K - 1; q > 0; --q) {   /* Fisher-Yates, counter-based draws */
        int64_t j = (int64_t)(rng(seed, ST_PERM, (uint64_t)q) % (uint64_t)(q + 1));
        int32_t t = perm[q]; perm[q] = perm[j]; perm[j] = t;
    }
    return 0;
}

static inline int64_t zipf_draw(const double* cdf, int64_t K, double u) {
    int64_t lo = 0, hi = K - 1;     /* first q with cdf[q] >= u */
    while (lo < hi) {
        int64_t mid = (lo + hi) >> 1;
        if (cdf[mid] >= u) hi = mid; else lo = mid + 1;
    }
    return lo;
}

/* Fill the columns of every row: deg = rowptr[i+1]-rowptr[i] distinct sorted
 * columns, drawn as described in the header.  Returns 0, or -1 if a row asks
 * for more than K distinct columns. */
int dg_powerlaw_fill(int64_t M, int64_t K, const int64_t* rowptr, double p_local, int64_t S,
                     const double* cdf, const int32_t* perm, uint64_t seed, int32_t* colidx) {
    int bad = 0;
    #pragma omp parallel for schedule(dynamic, 64) reduction(| : bad)
    for (int64_t i = 0; i < M; ++i) {
        int64_t d = rowptr[i + 1] - rowptr[i];
        if (d > K) { bad = 1; continue; }
        int32_t* buf = colidx + rowptr[i];
        int64_t base = (S * (i / S));
        if (base >= K) base = (K > S) ? K - S : 0;
        int64_t width = (base + S <= K) ? S : (K - base);
        int64_t have = 0;
        uint64_t ctr = 0;
        while (have < d) {
            int64_t need = d - have;
            /* scratch: draw into a temp and merge */
            int32_t* tmp = (int32_t*)malloc(sizeof(int32_t) * (size_t)(have + need));
            memcpy(tmp, buf, sizeof(int32_t) * (size_t)have);
            for (int64_t k = 0; k < need; ++k) {
                uint64_t x = rng(seed ^ (uint64_t)i * 0x9E3779B97F4A7C15ull, ST_COL, ctr++);
                double u = u01(x);
                double v = u01(mix64(x));
                int64_t c;
                if (u < p_local && width > 0) c = base + (int64_t)(v * (double)width);
                else c = perm[zipf_draw(cdf, K, v)];
                if (c >= K) c = K - 1;
                tmp[have + k] = (int32_t)c;
            }
            int64_t m = sort_unique(tmp, have + need);
            if (m > d) m = d;   /* cannot happen (unique of have+need <= d) but keep safe */
            memcpy(buf, tmp, sizeof(int32_t) * (size_t)m);
            have = m;
            free(tmp);
        }
    }
    return bad ? -1 : 0;
}

/* ------------------------------------------------------------------- G2 */
/* Row degrees: min(per_row, band width of row i); the n_out seeded outlier rows
 * get min(out_len, K).  Outlier row ids are written to out_rows[n_out]. */
int64_t dg_banded_degrees(int64_t M, int64_t K, int64_t per_row, int64_t half_band,
                          int64_t n_out, int64_t out_len, uint64_t seed,
                          int32_t* deg, int64_t* out_rows) {
    for (int64_t j = 0; j < n_out; ++j) {
        int64_t r;
        uint64_t ctr = 0;
        for (;;) {
            r = (int64_t)(rng(seed, ST_OUT, (uint64_t)(j * 1000003 + ctr++)) % (uint64_t)M);
            int dup = 0;
            for (int64_t q = 0; q < j; ++q) dup |= (out_rows[q] == r);
            if (!dup) break;
        }
        out_rows[j] = r;
    }
    int64_t total = 0;
    #pragma omp parallel for reduction(+ : total) schedule(static)
    for (int64_t i = 0; i < M; ++i) {
        int64_t lo = i - half_band < 0 ? 0 : i - half_band;
        int64_t hi = i + half_band > K - 1 ? K - 1 : i + half_band;
        int64_t w = hi - lo + 1;
        if (i >= K) w = 0;
        int64_t d = per_row < w ? per_row : w;
        if (d < 1 && K > 0) d = 1;
        deg[i] = (int32_t)d;
    }
    for (int64_t j = 0; j < n_out; ++j) deg[out_rows[j]] = (int32_t)(out_len < K ? out_len : K);
    for (int64_t i = 0; i < M; ++i) total += deg[i];
    return total;
}

int dg_banded_fill(int64_t M, int64_t K, const int64_t* rowptr, int64_t half_band,
                   int64_t n_out, const int64_t* out_rows, uint64_t seed, int32_t* colidx) {
    #pragma omp parallel for schedule(dynamic, 256)
    for (int64_t i = 0; i < M; ++i) {
        int64_t d = rowptr[i + 1] - rowptr[i];
        int32_t* buf = colidx + rowptr[i];
        int is_out = 0;
        for (int64_t j = 0; j < n_out; ++j) is_out |= (out_rows[j] == i);
        int64_t lo, w;
        if (is_out) { lo = 0; w = K; }
        else {
            int64_t c = i < K ? i : K - 1;
            lo = c - half_band < 0 ? 0 : c - half_band;
            int64_t hi = c + half_band > K - 1 ? K - 1 : c + half_band;
            w = hi - lo + 1;
        }
        int64_t have = 0;
        if (!is_out && d > 0) { buf[0] = (int32_t)(i < K ? i : K - 1); have = 1; }  /* diagonal */
        uint64_t ctr = 0;
        int32_t* tmp = (int32_t*)malloc(sizeof(int32_t) * (size_t)(d + 1));
        while (have < d) {
            int64_t need = d - have;
            memcpy(tmp, buf, sizeof(int32_t) * (size_t)have);
            for (int64_t k = 0; k < need; ++k) {
                uint64_t x = rng(seed ^ (uint64_t)i * 0x9E3779B97F4A7C15ull, ST_COL, ctr++);
                tmp[have + k] = (int32_t)(lo + (int64_t)(u01(x) * (double)w));
            }
            have = sort_unique(tmp, have + need);
            if (have > d) have = d;
            memcpy(buf, tmp, sizeof(int32_t) * (size_t)have);
        }
        free(tmp);
    }
    return 0;
}

/* ---------------------------------------------------------------- values */
/* out[p] = lo + (hi-lo)*u,  u ~ U[0,1) from rng(seed, stream, p) */
void dg_uniform_f32(uint64_t seed, uint64_t stream, int64_t n, float lo, float hi, float* out) {
    #pragma omp parallel for schedule(static)
    for (int64_t p = 0; p < n; ++p)
        out[p] = (float)((double)lo + (double)(hi - lo) * u01(rng(seed, stream, (uint64_t)p)));
}
/* out[p] = integer uniform in [lo, hi] */
void dg_int_f32(uint64_t seed, uint64_t stream, int64_t n, int64_t lo, int64_t hi, float* out) {
    uint64_t span = (uint64_t)(hi - lo + 1);
    #pragma omp parallel for schedule(static)
    for (int64_t p = 0; p < n; ++p)
        out[p] = (float)(lo + (int64_t)(rng(seed, stream, (uint64_t)p) % span));
}
/* out[p] = k/8 for an integer k uniform in [8*lo, 8*hi] (dyadic values) */
void dg_dyadic_f32(uint64_t seed, uint64_t stream, int64_t n, int64_t lo, int64_t hi, float* out) {
    uint64_t span = (uint64_t)(8 * (hi - lo) + 1);
    #pragma omp parallel for schedule(static)
    for (int64_t p = 0; p < n; ++p)
        out[p] = (float)((double)(8 * lo + (int64_t)(rng(seed, stream, (uint64_t)p) % span)) / 8.0);
}
