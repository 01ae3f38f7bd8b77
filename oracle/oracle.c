/*
 * oracle/oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously-correct CPU reference for the DTC-SpMM hot path.
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
 * reference legs may load this library.  It shares no code, header, table or
 * helper with the CUDA path (paper_conf_asplos_fan0024_b200/); neither side
 * includes or links the other.
 *
 * O1  oracle_spmm      C = A*B in FP64 (plain definition, §2.2
 *                      "C_{MxN} = A_{MxK} x B_{KxN}"), plus the error bound
 *                      Bound = |A|*|B| used by the tolerance (BASELINE.json
 *                      north_star).  Pinned by tests/test_oracle_pins.py
 *                      (dense brute force, identity, permutation, row sums).
 * O1s oracle_spmm_at   the same definition for a list of sampled (i, j).
 * O2  oracle_condense_* the ME-TCF reference condensation, step by step in the
 *                      paper's order: SGT "compressed towards the left side"
 *                      per 16-row window (§2.3) and the four
 *                      ME-TCF arrays (§4.2): RowWindowOffset,
 *                      TCOffset, TCLocalId (uint8), SparseAtoB, plus the
 *                      values array (reading C7).  Readings C3-C6
 *                      (ascending compaction order, id = row*8 + col, nnz in a
 *                      block by ascending id, -1 padding) are DESIGN.md's.
 *                      Pinned by decode round trip, closed forms and
 *                      brute-force dense-window condensation in the tests.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define WINDOW 16   /* BLOCK_HEIGHT; row window = 16 rows */
#define TCW 8       /* TC block = 16 x 8 */

int oracle_max_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
void oracle_set_threads(int n) {
#ifdef _OPENMP
    if (n > 0) omp_set_num_threads(n);
#else
    (void)n;
#endif
}

/* ------------------------------------------------------------------ O1 */
/* Rows [r0, r1) of C = A*B and Bound = |A|*|B| in FP64.
 * A: CSR (rowptr[M+1], colidx, vals as float32).  B: float32 row-major, ldb.
 * C, Bound: double, (r1-r0) x N, row stride N.  Bound may be NULL. */
int oracle_spmm(int64_t M, int64_t K, int64_t N, const int32_t* rowptr, const int32_t* colidx,
                const float* vals, const float* B, int64_t ldb, int64_t r0, int64_t r1,
                double* C, double* Bound) {
    (void)K;
    if (r0 < 0 || r1 > M || r0 > r1) return -1;
    #pragma omp parallel for schedule(dynamic, 256)
    for (int64_t i = r0; i < r1; ++i) {
        double* c = C + (i - r0) * N;
        double* bd = Bound ? Bound + (i - r0) * N : NULL;
        for (int64_t j = 0; j < N; ++j) c[j] = 0.0;
        if (bd) for (int64_t j = 0; j < N; ++j) bd[j] = 0.0;
        for (int64_t p = rowptr[i]; p < rowptr[i + 1]; ++p) {   /* sequential p order */
            const double a = (double)vals[p];
            const float* b = B + (int64_t)colidx[p] * ldb;
            for (int64_t j = 0; j < N; ++j) c[j] += a * (double)b[j];
            if (bd) {
                const double aa = fabs(a);
                for (int64_t j = 0; j < N; ++j) bd[j] += aa * fabs((double)b[j]);
            }
        }
    }
    return 0;
}

/* Sampled entries: C[rows[s], cols[s]] and its bound, s < count. */
int oracle_spmm_at(int64_t M, const int32_t* rowptr, const int32_t* colidx, const float* vals,
                   const float* B, int64_t ldb, int64_t count, const int64_t* rows,
                   const int64_t* cols, double* C, double* Bound) {
    #pragma omp parallel for schedule(dynamic, 64)
    for (int64_t s = 0; s < count; ++s) {
        int64_t i = rows[s], j = cols[s];
        double c = 0.0, bd = 0.0;
        if (i >= 0 && i < M)
            for (int64_t p = rowptr[i]; p < rowptr[i + 1]; ++p) {
                double a = (double)vals[p], b = (double)B[(int64_t)colidx[p] * ldb + j];
                c += a * b;
                bd += fabs(a) * fabs(b);
            }
        C[s] = c;
        if (Bound) Bound[s] = bd;
    }
    return 0;
}

/* ------------------------------------------------------------------ O2 */
static int cmp_i32(const void* a, const void* b) {
    int32_t x = *(const int32_t*)a, y = *(const int32_t*)b;
    return (x > y) - (x < y);
}

/* U = ascending unique column ids of window w's rows (windows of wh rows); returns |U| (U malloc'd). */
static int64_t window_unique(int64_t M, const int32_t* rowptr, const int32_t* colidx, int64_t wh,
                             int64_t w, int32_t** U_out) {
    int64_t rb = w * wh, re = rb + wh < M ? rb + wh : M;
    int64_t n = rowptr[re] - rowptr[rb];
    int32_t* U = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
    memcpy(U, colidx + rowptr[rb], sizeof(int32_t) * (size_t)n);
    qsort(U, (size_t)n, sizeof(int32_t), cmp_i32);
    int64_t u = 0;
    for (int64_t i = 0; i < n; ++i)
        if (u == 0 || U[i] != U[u - 1]) U[u++] = U[i];
    *U_out = U;
    return u;
}

/* rank of value x in ascending U (x must be present) */
static int64_t rank_of(const int32_t* U, int64_t u, int32_t x) {
    int64_t lo = 0, hi = u;
    while (lo < hi) {
        int64_t mid = (lo + hi) >> 1;
        if (U[mid] < x) lo = mid + 1; else hi = mid;
    }
    return lo;
}

/* Steps 1-2: RowWindowOffset[W+1] (int32). Returns NumTCBlock T, or -1.
 * wh = rows per window: 16 = the paper's BLOCK_HEIGHT; 32 = the tall windows of the
 * NEXT-2 layout (reading C2b: the same SGT condensation applied to 32-row windows). */
int64_t oracle_condense_count_wh(int64_t M, const int32_t* rowptr, const int32_t* colidx, int64_t wh,
                                 int32_t* row_window_offset) {
    int64_t W = (M + wh - 1) / wh;
    int64_t* nb = (int64_t*)malloc(sizeof(int64_t) * (size_t)(W > 0 ? W : 1));
    #pragma omp parallel for schedule(dynamic, 16)
    for (int64_t w = 0; w < W; ++w) {
        int32_t* U;
        int64_t u = window_unique(M, rowptr, colidx, wh, w, &U);
        nb[w] = (u + TCW - 1) / TCW;          /* nTC_w = ceil(u_w / 8) */
        free(U);
    }
    int64_t acc = 0;
    row_window_offset[0] = 0;
    for (int64_t w = 0; w < W; ++w) {
        acc += nb[w];
        if (acc > INT32_MAX) { free(nb); return -1; }
        row_window_offset[w + 1] = (int32_t)acc;
    }
    free(nb);
    return acc;
}

/* Steps 3-5: SparseAtoB[8T], TCOffset[T+1], TCLocalId[nnz], TCValues[nnz].
 * vals/tc_values are opaque elements of elem_size bytes (fp32 or fp16). */
int oracle_condense_fill_wh(int64_t M, const int32_t* rowptr, const int32_t* colidx, int64_t wh,
                            const void* vals, int64_t elem_size, const int32_t* row_window_offset,
                            int32_t* tc_offset, uint8_t* tc_local_id, int32_t* sparse_a_to_b,
                            void* tc_values) {
    int64_t W = (M + wh - 1) / wh;
    const uint8_t* vin = (const uint8_t*)vals;
    uint8_t* vout = (uint8_t*)tc_values;
    int bad = 0;
    #pragma omp parallel for schedule(dynamic, 16) reduction(| : bad)
    for (int64_t w = 0; w < W; ++w) {
        int32_t* U;
        int64_t u = window_unique(M, rowptr, colidx, wh, w, &U);
        int64_t blk0 = row_window_offset[w];
        int64_t nb = row_window_offset[w + 1] - blk0;
        if (nb != (u + TCW - 1) / TCW) { bad = 1; free(U); continue; }
        /* step 3: SparseAtoB = U[8b .. 8b+7], -1 padded */
        for (int64_t b = 0; b < nb; ++b)
            for (int64_t i = 0; i < TCW; ++i) {
                int64_t k = b * TCW + i;
                sparse_a_to_b[(blk0 + b) * TCW + i] = k < u ? U[k] : -1;
            }
        /* step 4: traverse the window's nnz in CSR order, bucket by block */
        int64_t rb = w * wh, re = rb + wh < M ? rb + wh : M;
        int64_t* cnt = (int64_t*)calloc((size_t)(nb + 1), sizeof(int64_t));
        for (int64_t r = rb; r < re; ++r)
            for (int64_t p = rowptr[r]; p < rowptr[r + 1]; ++p)
                cnt[rank_of(U, u, colidx[p]) / TCW]++;
        /* step 5: emit buckets b = 0..nb-1 in order; TCOffset after each */
        int64_t start = rowptr[rb];
        int64_t* cur = (int64_t*)malloc(sizeof(int64_t) * (size_t)(nb + 1));
        int64_t acc = start;
        for (int64_t b = 0; b < nb; ++b) {
            tc_offset[blk0 + b] = (int32_t)acc;
            cur[b] = acc;
            acc += cnt[b];
        }
        for (int64_t r = rb; r < re; ++r)
            for (int64_t p = rowptr[r]; p < rowptr[r + 1]; ++p) {
                int64_t k = rank_of(U, u, colidx[p]);
                int64_t b = k / TCW;
                int64_t id = (r - rb) * TCW + (k % TCW);      /* id = row_in_window*8 + col_in_block */
                int64_t dst = cur[b]++;                        /* stable: CSR order within bucket */
                tc_local_id[dst] = (uint8_t)id;
                memcpy(vout + dst * elem_size, vin + p * elem_size, (size_t)elem_size);
            }
        free(cur); free(cnt); free(U);
    }
    int64_t T = row_window_offset[W];
    tc_offset[T] = rowptr[M];
    return bad ? -1 : 0;
}

/* The paper's ME-TCF: 16-row windows. */
int64_t oracle_condense_count(int64_t M, const int32_t* rowptr, const int32_t* colidx,
                              int32_t* row_window_offset) {
    return oracle_condense_count_wh(M, rowptr, colidx, WINDOW, row_window_offset);
}
int oracle_condense_fill(int64_t M, const int32_t* rowptr, const int32_t* colidx,
                         const void* vals, int64_t elem_size, const int32_t* row_window_offset,
                         int32_t* tc_offset, uint8_t* tc_local_id, int32_t* sparse_a_to_b,
                         void* tc_values) {
    return oracle_condense_fill_wh(M, rowptr, colidx, WINDOW, vals, elem_size, row_window_offset, tc_offset,
                                   tc_local_id, sparse_a_to_b, tc_values);
}
