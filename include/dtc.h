/*
 * dtc.h -- C ABI of libdtc.so: the DTC-SpMM hot path on B200 (sm_100a).
 *
 * Operation: general unstructured SpMM  C(MxN) = A(MxK) * B(KxN)  with A sparse
 * (§2.2), B and C dense row-major (§4.4.1), computed
 * on tensor cores over the memory-efficient tensor-core format ME-TCF
 * (§4.2) built from CSR on the GPU (§6).
 * A fixed A is converted once and reused across many SpMM calls.
 *
 * Conventions (all entry points):
 *  - Every function returns a dtc_status_t (0 = DTC_OK, negative = error).  No
 *    exception or abort crosses the ABI; dtc_last_error() returns a thread-local
 *    message with detail.
 *  - Pointers are DEVICE pointers unless the name/comment says host.  Streams
 *    are passed as `void*` holding a cudaStream_t (NULL = legacy default stream).
 *  - The caller owns CSR, B and C.  The library owns everything reachable from a
 *    handle (format arrays, schedule, workspaces) until *_destroy.
 *  - There is no CPU fallback: without a CUDA device every compute call returns
 *    DTC_ERR_CUDA.
 */
#ifndef DTC_H_
#define DTC_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    DTC_OK = 0,
    DTC_ERR_INVALID = -1,     /* bad argument / malformed rowptr              */
    DTC_ERR_UNSORTED = -2,    /* CSR columns not ascending within a row       */
    DTC_ERR_DUPLICATE = -3,   /* repeated column within a row                 */
    DTC_ERR_RANGE = -4,       /* column index outside [0, K)                  */
    DTC_ERR_OOM = -5,         /* device allocation failed                     */
    DTC_ERR_CUDA = -6,        /* CUDA runtime error (incl. no device)         */
    DTC_ERR_NCCL = -7,        /* NCCL error                                   */
    DTC_ERR_UNSUPPORTED = -8  /* valid request this build does not handle     */
} dtc_status_t;

/* Value / operand precision.
 * DTC_TF32: A values and B are fp32 in memory; A is rounded to TF32 (cvt.rna)
 *           when staged, B is fed to the tensor core as fp32 bits (TF32 truncation);
 *           fp32 accumulation (error budget in DESIGN.md C13).
 * DTC_FP16: A values and B are fp16 in memory; fp32 accumulation; C is fp32.   */
typedef enum { DTC_TF32 = 0, DTC_FP16 = 1 } dtc_dtype_t;

/* Canonical CSR input (device pointers): rowptr int32[M+1] with rowptr[0]=0,
 * rowptr[M]=nnz, non-decreasing; colidx int32[nnz] strictly increasing within a
 * row and in [0,K); vals[nnz] of `dtype` (fp32 or fp16).  nnz < 2^31.
 * Explicit zeros are structural non-zeros and are kept. */
typedef struct {
    int64_t M, K, nnz;
    const int32_t* rowptr;
    const int32_t* colidx;
    const void* vals;
    int32_t dtype;            /* dtc_dtype_t */
} dtc_csr_t;

typedef struct dtc_format* dtc_handle_t;   /* opaque, library-owned */

/* Borrowed device views of the ME-TCF arrays, valid until
 * dtc_format_destroy:
 *   row_window_offset int32[num_windows+1]  start TC block of each 16-row window
 *   tc_offset         int32[T+1]            start of each TC block in tc_local_id
 *   tc_local_id       uint8[nnz]            row_in_window*8 + col_in_block (<128)
 *   sparse_a_to_b     int32[8T]             original column of each block column, -1 pad
 *   tc_values         dtype[nnz]            values aligned with tc_local_id
 *   units             int32[8*num_units]    F4 work units {wb, we, bb, be, split_id, piece,
 *                                            npieces, slot_base} (see dtc_format_export) */
typedef struct {
    int64_t M, K, nnz, num_windows, num_tc_blocks, num_units, num_split_windows;
    int32_t dtype;
    int32_t unit_blocks;
    int32_t window_rows;   /* 16 (ME-TCF) or 32 (dtc_build_opts_t.window_rows) */
    const int32_t* row_window_offset;
    const int32_t* tc_offset;
    const uint8_t* tc_local_id;
    const int32_t* sparse_a_to_b;
    const void* tc_values;
    const int32_t* units;
} dtc_format_view_t;

/* Build options (zero-initialised = defaults; window_order, n_hint, selector documented at the fields).
 *   unit_blocks  target TC blocks per work unit (F4); 0 = auto from T, W and the SM count
 *   dedup_path   F1 per-window dedup: 0 auto, 1 force smem sort, 2 force chunked bitmap
 *                (both produce bit-identical formats; exposed for tests)
 *   guided       F4 tail: units of U/2 over the last ~half wave: 1 = on, -1 = off, 0 = auto (on
 *                when T < 8 waves x 6 CTAs x SMs x U, i.e. short launches; +5% on the arxiv-shaped c2) */
typedef struct {
    int32_t unit_blocks;
    int32_t dedup_path;
    int32_t guided;
    int32_t window_order;   /* F4 unit order: 0 = pieces of split windows first, then whole-window
                               units (default; the split fixups overlap the launch instead of
                               forming its tail), 1 = strict window order.  Same results. */
    /* optional row permutation (DEVICE int32[M], new row -> original row, a bijection):
     * the library condenses the permuted matrix and dtc_spmm still writes C in the
     * ORIGINAL row order (e.g. the TCA order from dtc_tca_reorder).  NULL = identity.
     * Not a permutation -> DTC_ERR_INVALID. */
    const int32_t* row_perm;
    /* B200 Selector (NEXT-4, dtc_selector_plan): with unit_blocks = 0 and selector = 1, F4 takes the
     * unit size and guided tail whose simulated launch for N = n_hint columns (0 = 128) is shortest;
     * selector = 0 keeps the fixed rule (U = clamp(2T/W, 64, 256), at most T/(24 SMs); guided as above).
     * With selector = 1 or 2, window_rows = 0 and a TF32 matrix whose gathered rows are >= 1 KB
     * (n_hint x 4 >= 1024), it also picks the window height: 32 rows (NEXT-2) when that lowers the TC
     * blocks to <= 0.65 of the 16-row count (F0-F2 run at both heights first); selector = 2 picks
     * only the window height and keeps the fixed unit-size rule (the simulated U plan ignores L2
     * locality and lost 4% on the products-shaped c5).
     * Same C either way (within tolerance; integer inputs bit-exact). */
    int32_t n_hint;
    int32_t selector;
    /* transpose = 1: condense A^T (K x M) instead of A -- the rows of A^T are A's columns, in the
     * canonical order (A's CSR is validated first; then a GPU radix sort by (column, row) gives A^T's
     * CSR) -- e.g. the handle for the GCN backward dH = A^T dAH (NEXT-3).  Not combinable with
     * row_perm (INVALID). */
    int32_t transpose;
    /* window_rows = 32: condense with 32-row windows (TC blocks of 32 x 8, local ids 0..255 still in
     * uint8, SparseAtoB per 32-row window) -- the NEXT-2 layout in which two consecutive 16-row
     * windows gather their shared B rows once; 0 or 16 = the paper's ME-TCF.  The
     * view's arrays then describe 32-row windows; dtc_spmm computes the same C. */
    int32_t window_rows;
} dtc_build_opts_t;

/* F0-F4: validate CSR, condense into ME-TCF and build the work-unit schedule on
 * the GPU.  Stream-ordered; blocks on `stream`
 * twice (to read NumTCBlock + the validation flag, and the unit count) in
 * order to size allocations.  On error *out is NULL and nothing leaks.
 * Errors: INVALID (null/negative sizes, malformed rowptr), UNSORTED, DUPLICATE,
 * RANGE, OOM, CUDA. */
int dtc_format_build(const dtc_csr_t* csr, void* stream, dtc_handle_t* out);
int dtc_format_build_ex(const dtc_csr_t* csr, const dtc_build_opts_t* opts, void* stream,
                        dtc_handle_t* out);

/* Fill *view with borrowed device pointers and sizes.  INVALID if h or view is NULL. */
int dtc_format_query(dtc_handle_t h, dtc_format_view_t* view);

/* Copy the ME-TCF arrays to HOST buffers (any pointer may be NULL to skip it):
 * rwo int32[W+1], tco int32[T+1], lid uint8[nnz], atob int32[8T],
 * vals dtype[nnz], units int32[8*num_units].  Synchronous. */
int dtc_format_export(dtc_handle_t h, int32_t* rwo, int32_t* tco, uint8_t* lid, int32_t* atob,
                      void* vals, int32_t* units);

/* S1-S5: C := A*B (kernel design PAPER.md:260-333, re-designed for
 * sm_100a).  B: device, K x N row-major with row stride ldb >= N, dtype of the
 * handle.  C: device fp32, M x N row-major with ldc >= N; every element of the
 * M x N region is overwritten (empty rows -> 0).  N >= 1.  Asynchronous on
 * `stream`; deterministic (bit-identical run to run).  16-byte aligned B/C with
 * ldb, ldc, N multiples of 16/sizeof(elt) take the vector path, anything else the
 * scalar path.  Concurrent dtc_spmm calls on ONE handle must be stream-ordered
 * (they share the split-window workspace).  Errors: INVALID, CUDA, OOM. */
int dtc_spmm(dtc_handle_t h, const void* B, int64_t N, int64_t ldb, float* C, int64_t ldc,
             void* stream);

/* End-to-end variant with HOST buffers: copies B (host, K x N, ldb) to a
 * library-owned device buffer, runs dtc_spmm, copies C back to host (M x N,
 * ldc) and synchronises `stream`.  Pinned host memory gives full PCIe/C2C rate.
 * Calls of >= 8 MB are pipelined over column chunks (C(:, cols) depends only on B(:, cols)):
 * the copy-in of chunk j+1 overlaps chunk j's kernel and copy-out on library-owned streams;
 * the result is bit-identical to one dtc_spmm over all N columns.  Chunks: up to 4, each >= 512 B
 * of a B row (>= 256 B when the format is smaller than B).  When the format is larger than B (long kernels) and C_host is pinned and
 * mapped, the kernel stores C straight into C_host (no copy-out).  DTC_OPT_HOST_CHUNKS and
 * DTC_OPT_HOST_ZERO_COPY override both choices; DTC_OPT_LAST_HOST_MODE reports them.  The caller
 * guarantees B_host holds K rows of ldb elements of the handle's dtype and C_host M rows of ldc
 * floats (the library cannot check host extents).  On error no copy is left running against the
 * host buffers. */
int dtc_spmm_host(dtc_handle_t h, const void* B_host, int64_t N, int64_t ldb, float* C_host,
                  int64_t ldc, void* stream);

/* Streaming variant of dtc_spmm_host for a sequence of products with the same A (e.g. GNN inference
 * over many feature batches): enqueues the copy-in of B_host, the kernel and the copy-out of C
 * (or zero-copy C, as above) and returns WITHOUT waiting.  The library keeps two device staging sets:
 * call j's copy-in waits, on the device, only for call j-2's kernel, so the copy-in of call j+1
 * overlaps the kernel of call j and the copy-out of call j-1 (PCIe is full duplex).  B_host must not
 * change and C_host must not be read until dtc_spmm_host_wait(h) returns.  Each call computes
 * exactly what dtc_spmm computes.  Errors: as dtc_spmm_host (checked at enqueue). */
int dtc_spmm_host_async(dtc_handle_t h, const void* B_host, int64_t N, int64_t ldb, float* C_host,
                        int64_t ldc, void* stream);
/* Wait for every dtc_spmm_host_async call enqueued on h.  Errors: INVALID, CUDA. */
int dtc_spmm_host_wait(dtc_handle_t h);

/* Number of kernels dtc_spmm launches per call (for launch accounting). */
int dtc_spmm_launches_per_call(void);

/* Per-handle launch options (defaults are the measured best).  Options change how
 * dtc_spmm / dtc_spmm_host run, never what they compute: every setting gives the same C within
 * the north_star tolerance, and the padded-path options give bit-identical C (tested).
 *   DTC_OPT_KERNEL         0 auto = TMA padded-row kernel (k_spmm_pad) where TMA can describe B
 *                          (16-byte aligned base and row pitch), else the register-gather kernel
 *                          (k_spmm_ldg, the paper's FetchSparse/VFetchDense structure);
 *                          1 forces the register-gather kernel; 4 requests the padded kernel
 *                          (it still falls back where TMA cannot describe B).
 *   DTC_OPT_PERSISTENT     padded kernel: 1 = one wave of CTAs drawing F4 units from an atomic
 *                          counter, largest first; 0 = one CTA per unit (default).
 *   DTC_OPT_FIRST_RECORDS  padded kernel: 1 = per-unit side records of the first batch (default).
 *   DTC_OPT_HOST_CHUNKS    dtc_spmm_host column chunks, 0 = auto, 1..16.
 *   DTC_OPT_HOST_ZERO_COPY dtc_spmm_host stores C straight into pinned mapped C_host:
 *                          -1 = auto (when the format is larger than B), 0 = off, 1 = on.
 *   DTC_OPT_SLICE_BYTES    padded kernel row slice per gather4 op: 0 auto (1024 when a B row holds
 *                          >= 1 KB, 256 when it holds <= 256 B, else 512), 512 or 1024.
 *   DTC_OPT_LAST_KERNEL    read-only: kernel the last dtc_spmm ran (1 register gather, 4 padded).
 *   DTC_OPT_LAST_HOST_MODE read-only: last dtc_spmm_host: 2 * column chunks + (1 if C was stored
 *                          zero-copy into host memory, i.e. no device-to-host copy).
 * Not synchronised against concurrent calls on the same handle (like dtc_spmm itself).
 * Errors: INVALID (null handle, unknown option, value out of range, read-only option). */
typedef enum {
    DTC_OPT_KERNEL = 1,
    DTC_OPT_PERSISTENT = 2,
    DTC_OPT_FIRST_RECORDS = 3,
    DTC_OPT_HOST_CHUNKS = 4,
    DTC_OPT_HOST_ZERO_COPY = 5,
    DTC_OPT_SLICE_BYTES = 6,
    DTC_OPT_LAST_KERNEL = 100,
    DTC_OPT_LAST_HOST_MODE = 101,
    DTC_OPT_GUIDED = 102,            /* read-only: 1 if F4 cut a guided tail */
    DTC_OPT_PLAN_MAKESPAN_NS = 103   /* read-only: the Selector's simulated makespan (ns), 0 = fixed rule */
} dtc_option_t;
int dtc_format_set_option(dtc_handle_t h, int32_t option, int64_t value);
int dtc_format_get_option(dtc_handle_t h, int32_t option, int64_t* value);

/* Diagnostics (the paper's per-SM busy/idle methodology, Fig. 3 P:152-160 / Fig. 15):
 * while enabled, each CTA of the padded kernel launched for handle h writes 8 int64 to
 * dev_buf[cta*8 ..]: {cta, smid, t_start, t_first_issue, t_first_data, t_consumer_done,
 * num_tc_blocks, t_producer_done}, times in ns of the %globaltimer.  dev_buf is a caller-owned
 * device buffer of capacity_ctas*8 int64 that must outlive its use; launches with more CTAs than
 * capacity_ctas are not traced.  capacity_ctas = 0 disables.  Errors: INVALID. */
int dtc_format_set_trace(dtc_handle_t h, void* dev_buf, int64_t capacity_ctas);

void dtc_format_destroy(dtc_handle_t h);   /* NULL-safe; frees all device memory */

/* ------------------------------------------------------------ reordering (NEXT-1)
 * TCU-Cache-Aware reordering, §4.3 Alg. 1 (optional HOST
 * preprocessing): MinHash-LSH row pairs -> priority queue by Jaccard -> row clusters
 * of BLOCK_HEIGHT = 16 rows (Hierarchy I), then the same over row clusters into
 * clusters of sm_num clusters (Hierarchy II, L2 locality), then Reid.  HOST inputs:
 * canonical CSR pattern rowptr[M+1], colidx[nnz].  Output perm[M] (host): new row ->
 * original row, to pass as dtc_build_opts_t.row_perm (after copying to the device).
 * Deterministic (readings DESIGN.md T1-T8).  Errors: INVALID, OOM. */
int dtc_tca_reorder(int64_t M, int64_t K, const int32_t* rowptr_host, const int32_t* colidx_host,
                    int32_t sm_num, int32_t* perm_host);

/* dtc_tca_reorder, then keep it only if it pays: NumTCBlock of the reordered and of
 * the original row order are counted on the host; when the reordering does not lower it (e.g. a
 * banded matrix already in its best order) perm is set to the identity.  T_identity, T_reordered
 * (the counts) and applied (1 if perm is the TCA order) may each be NULL.  Errors: as above. */
int dtc_tca_reorder_checked(int64_t M, int64_t K, const int32_t* rowptr_host, const int32_t* colidx_host,
                            int32_t sm_num, int32_t* perm_host, int64_t* T_identity, int64_t* T_reordered,
                            int32_t* applied);

/* ------------------------------------------------------------ GraphConv (NEXT-3)
 * One GCN layer, §5.4 Eq. (2): Y = act((A x H) x W + b), in the
 * paper's order: AH = A*H by dtc_spmm (this library's kernel), then the dense
 * AH*W with bias and activation fused into a cuBLASLt TF32 GEMM epilogue (a plain
 * library GEMM; FP32 accumulate).  All pointers device, row-major, dense:
 *   H    K x F_in, dtype of the handle (fp32 for TF32 handles, fp16 for FP16);
 *   W    F_in x F_out fp32;  bias F_out fp32 or NULL;  act DTC_ACT_NONE | DTC_ACT_RELU;
 *   AH   M x F_in fp32, caller-owned workspace (holds A*H on return);
 *   Y    M x F_out fp32, overwritten.
 * Asynchronous on `stream`.  Errors: INVALID, UNSUPPORTED, OOM, CUDA. */
typedef enum { DTC_ACT_NONE = 0, DTC_ACT_RELU = 1 } dtc_act_t;
int dtc_graphconv(dtc_handle_t h, const void* H, int64_t F_in, const float* W, int64_t F_out,
                  const float* bias, int32_t act, float* AH, float* Y, void* stream);
/* Kernels one dtc_graphconv launches at least (SpMM + GEMM; cuBLASLt may add a reduction). */
int dtc_graphconv_launches_per_call(void);

/* Backward of one GraphConv layer Y = act(Z), Z = (A x H) x W + b (chain rule on Eq. (2)):
 *   dZ  = dY * act'(Z)   (ReLU: 1 where Y > 0, else 0 -- the mask is read from Y; identity: dY)
 *   dW  = AH^T dZ        (F_in x F_out)      cuBLASLt TF32, FP32 accumulate
 *   db  = sum_rows dZ    (F_out; may be NULL) deterministic fixed-order reduction
 *   dAH = dZ W^T         (M x F_in)          cuBLASLt TF32
 *   dH  = A^T dAH        (K x F_in; may be NULL to skip) -- DTC-SpMM on ht, the ME-TCF of A^T built
 *                        by dtc_format_build_ex with opts.transpose = 1 (TF32 handles only)
 * AH, Y are the forward's; dZ (M x F_out) is caller workspace and may alias dY.  All device fp32
 * row-major.  Errors: INVALID (shapes/handles), UNSUPPORTED (FP16 A^T), OOM, CUDA. */
int dtc_graphconv_backward(dtc_handle_t h, dtc_handle_t ht, const float* AH, const float* W, int64_t F_in,
                           int64_t F_out, int32_t act, const float* Y, const float* dY, float* dZ, float* dW,
                           float* db, float* dAH, float* dH, void* stream);

/* Training-step helpers for a GCN on top of the layer (NEXT-3):
 * dtc_softmax_xent: loss (device scalar) = mean_i [log sum_c exp(z_ic) - z_i,label_i] over M rows of
 * logits (M x num_classes, fp32), dlogits = (softmax(z_i) - onehot(label_i)) / M; labels int32[M] in
 * [0, num_classes) (INVALID otherwise).  Synchronises `stream` (to report bad labels).
 * dtc_sgd_update: param[i] -= lr * grad[i], i < n.  Errors: INVALID, OOM, CUDA. */
int dtc_softmax_xent(const float* logits, const int32_t* labels, int64_t M, int64_t num_classes, float* loss,
                     float* dlogits, void* stream);
int dtc_sgd_update(float* param, const float* grad, int64_t n, float lr, void* stream);

/* ------------------------------------------------------------ Selector (NEXT-4, diagnostic)
 * Simulation-based Selector, §4.5.2, Eq. (1), Fig. 10.  HOST, pure
 * (no GPU needed).  rwo_host: RowWindowOffset int32[num_windows+1] (host copy, e.g.
 * from dtc_format_export).  Simulates the base kernel (one thread block per window,
 * length nTC_w) under the TB-scheduling model sm = 2(b mod S/2) + (floor(b/(S/2)) mod 2)
 * (Eq. (1) with 64 -> S/2; reading C23) with `occupancy` resident blocks per
 * SM, each SM running its blocks in index order on the first freed slot.  Outputs
 * (each may be NULL): makespan_base = max over SMs of the last finish time (in TC
 * blocks), makespan_balanced = NumTCBlocks / (num_sms * occupancy), ar = base /
 * balanced (1 when T = 0).  The paper launches its balanced kernel when ar > 1.2;
 * libdtc always runs TC-block-balanced units, so this is a report.
 * Errors: INVALID (odd or < 2 num_sms, occupancy outside 1..1024, non-monotone rwo). */
int dtc_selector_ar(const int32_t* rwo_host, int64_t num_windows, int32_t num_sms, int32_t occupancy,
                    double* makespan_base, double* makespan_balanced, double* ar);

/* ------------------------------------------------------------ B200 Selector (NEXT-4)
 * The paper's Selector (§4.5.2) simulates its base kernel's thread-block
 * schedule to decide whether balancing pays.  libdtc always runs TC-block-balanced F4 units, so
 * the retargeted Selector decides how to cut them: it simulates, for each candidate unit size U
 * (and with/without the guided tail), the launch of exactly the units F4 would emit -- dispatched
 * in order onto num_sms x occupancy resident-CTA slots, each unit holding its slot for
 * cta_ns + block_ns * nb (+ fixup_ns * (G + ceil(np/G)) on the last piece of a window split into
 * np pieces, G = ceil(sqrt(np)) or np if np <= 4) -- and keeps the shortest makespan (ties: larger U).
 * dtc_format_build_ex runs it when opts->selector = 1 and opts->unit_blocks = 0. */
typedef struct {
    int32_t num_sms;      /* SMs (148 on B200) */
    int32_t occupancy;    /* resident CTAs per SM of the kernel that will run (measured) */
    double cta_ns;        /* slot time of a CTA beyond its blocks (startup + epilogue) */
    double block_ns;      /* slot time per TC block */
    double fixup_ns;      /* per dependent partial load of a split-window fixup */
} dtc_sched_model_t;
typedef struct {
    int32_t unit_blocks;  /* U */
    int32_t guided;       /* 1 = guided tail (units of U/2 over the last ~4U blocks per SM) */
    int64_t num_units;    /* units (CTAs per column group) of the plan; -1 = not evaluated */
    double makespan_ns;   /* simulated makespan; -1 = not evaluated */
} dtc_plan_t;

/* Default B200 model for dtype and N on the CURRENT device: occupancy measured with
 * cudaOccupancyMaxActiveBlocksPerMultiprocessor on the kernel dtc_spmm would launch for N,
 * cta_ns 2500, block_ns = occupancy x 8 x (CTA columns) x elt / (62.8 B/ns per SM, the measured
 * gather4 rate), fixup_ns 1000.  Errors: INVALID, CUDA (no device). */
int dtc_sched_model(int32_t dtype, int64_t N, dtc_sched_model_t* m);

/* HOST, pure: plan F4 for RowWindowOffset rwo_host[W+1].  cand_u[ncand] candidate unit sizes (>= 8;
 * NULL / 0 = {16,24,32,48,64,96,128,192,256,384,512}); guided: 0 = try both, 1 = only with, -1 =
 * only without the guided tail.  plans (may be NULL) receives 2*ncand entries, plan k = candidate
 * k/2 with guided = k&1 (excluded plans have makespan -1); best receives the winner.
 * Errors: INVALID (bad model, non-monotone rwo, candidate < 8). */
int dtc_selector_plan(const int32_t* rwo_host, int64_t num_windows, const dtc_sched_model_t* m,
                      const int32_t* cand_u, int32_t ncand, int32_t guided, dtc_plan_t* plans,
                      dtc_plan_t* best);

/* HOST, pure: simulated makespan (ns) of an explicit unit list (units_host int32[8*nu] in the
 * dtc_format_export layout, dispatched in the given order) under model m.  Errors: INVALID. */
int dtc_selector_simulate(const int32_t* units_host, int64_t nu, const dtc_sched_model_t* m,
                          double* makespan_ns);

/* ------------------------------------------------------------ distributed
 * One process per GPU (north_star).  Row windows are partitioned across ranks
 * into contiguous ranges balanced by TC-block count; every rank needs all of B,
 * which the root broadcasts with NCCL; C can be all-gathered. */
typedef struct dtc_dist* dtc_dist_t;

/* HOST, pure: split windows [0,W) into `world` contiguous ranges at the smallest
 * w with rwo[w] >= r*T/world (r = 1..world-1).  w_begin int64[world+1].
 * Callable without a GPU.  INVALID on bad sizes. */
int dtc_partition_windows(const int32_t* rwo_host, int64_t num_windows, int32_t world,
                          int64_t* w_begin);

/* Write a fresh 128-byte NCCL unique id to out128 (host). */
int dtc_nccl_unique_id(void* out128);

/* Collective over `world` ranks: count the FULL csr's TC blocks per window (F0-F2 only; device
 * pointers on this rank's GPU) to find the window partition, then build this rank's local ME-TCF
 * from its CSR row slice.  nccl_id (host, 128 B, identical on all ranks) may be
 * NULL for a communicator-less local shard (single-GPU shard tests). */
int dtc_dist_create(const dtc_csr_t* csr_full, int32_t rank, int32_t world, const void* nccl_id,
                    void* stream, dtc_dist_t* out);

/* This rank's C rows [row_begin, row_end) and its local format handle (borrowed). */
int dtc_dist_query(dtc_dist_t d, int64_t* row_begin, int64_t* row_end, dtc_handle_t* local);

/* B: device K x N (ldb = N), read on `root` only (other ranks may pass NULL; their B is not
 * written).  The root packs B into column chunks (dtc_dist_chunks) of a library-owned buffer and
 * broadcasts them with NCCL on a library stream while every rank's kernel computes the previous
 * chunk's columns -- C(:, cols) depends only on B(:, cols), so C is bit-identical to one dtc_spmm
 * over all N columns.  C: device fp32; if gather_c, M x N (ldc = N) and every rank receives all
 * rows (grouped NCCL broadcasts per owner after the last chunk); else this rank's
 * (row_end-row_begin) x N rows.  Without a communicator (nccl_id NULL) B must be resident and the
 * call is a local dtc_spmm.  Stream-ordered on `stream`.  Errors: INVALID, NCCL, CUDA, OOM. */
int dtc_spmm_dist(dtc_dist_t d, void* B, int32_t root, int64_t N, float* C, int32_t gather_c,
                  void* stream);

/* HOST, pure: the column chunks of dtc_spmm_dist for K x N (elt bytes per element): widths are
 * multiples of 32 columns, at most max_chunks (0 = 4, capped at 8), each >= 128 KB of B.
 * col_begin int64[chunks+1].  Returns the number of chunks (>= 1) or INVALID. */
int dtc_dist_chunks(int64_t K, int64_t N, int32_t elt, int32_t max_chunks, int64_t* col_begin);

/* Override the chunk count of dtc_spmm_dist (0 = auto, 1 = unpipelined, up to 8).  Errors: INVALID. */
int dtc_dist_set_chunks(dtc_dist_t d, int32_t chunks);

void dtc_dist_destroy(dtc_dist_t d);

/* ------------------------------------------------------------ diagnostics */
const char* dtc_status_string(int status);
const char* dtc_last_error(void);
/* Library build string (arch, version). */
const char* dtc_version(void);

#ifdef __cplusplus
}
#endif
#endif /* DTC_H_ */
