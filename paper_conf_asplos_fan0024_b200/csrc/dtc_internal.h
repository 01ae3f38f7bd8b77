// dtc_internal.h -- private declarations shared by the libdtc.so translation units.
#pragma once

#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
#include <string>
#include <vector>

#include "../../include/dtc.h"

namespace dtc {

constexpr int kWindow = 16;   // BLOCK_HEIGHT
constexpr int kTcw = 8;       // TC block width

// Work-unit record (F4).  Unit u covers TC blocks [bb, be) and the C rows of
// windows [wb, we).  split_id >= 0 marks one piece of a window that was split
// across several units: its partial goes to workspace slot (slot_base + piece)
// and the last arriving piece sums slots in order (deterministic fixup).
struct Unit {
    int32_t wb, we, bb, be;
    int32_t split_id, piece, npieces, slot_base;
};
static_assert(sizeof(Unit) == 32, "unit record is 8 x int32");

// Per-handle launch options (dtc_format_set_option; include/dtc.h DTC_OPT_*).
struct Options {
    int32_t kernel = 0;          // 0 auto, 1 register gather, 4 TMA padded rows
    int32_t persistent = 0;      // padded path: one wave of CTAs drawing units
    int32_t first_records = 1;   // padded path: per-unit first-batch side records
    int32_t host_chunks = 0;     // dtc_spmm_host column chunks, 0 = auto
    int32_t host_zc = -1;        // dtc_spmm_host zero-copy C: -1 auto, 0 off, 1 on
    int32_t slice_bytes = 0;     // padded path: 0 auto, 512 or 1024
};

}  // namespace dtc

struct dtc_format {
    int64_t M = 0, K = 0, nnz = 0, W = 0, T = 0;
    int32_t dtype = 0;
    int32_t window_h = 16;            // rows per window: 16 (ME-TCF) or 32 (tall windows, NEXT-2)
    int32_t unit_blocks = 0;
    int32_t guided = 0;               // F4 guided tail in use
    double plan_makespan_ns = 0.0;    // Selector's simulated makespan of the chosen plan (0 = rule)
    int device = 0;
    int32_t* rwo = nullptr;      // [W+1]
    int32_t* tco = nullptr;      // [T+1]
    uint8_t* lid = nullptr;      // [nnz]
    int32_t* atob = nullptr;     // [8T]
    void* vals = nullptr;        // [nnz] fp32 / fp16
    // kernel-side index derived from TCLocalId (not part of ME-TCF): 128-bit (window_h = 32: 256-bit)
    // occupancy of each TC block, bit id = local id.  TCValues[TCOffset[b] + popcount(mask below id)] is the value
    // at id (C5: ascending local id), so a lane builds its A fragment without a shared-memory scatter.
    uint32_t* mask = nullptr;    // [4T] (window_h = 32: [8T])
    // F4 schedule
    int64_t num_units = 0;
    int64_t num_split = 0;       // split windows
    int64_t num_slots = 0;       // total split pieces
    dtc::Unit* units = nullptr;
    // split fixup state: counters [num_split * max_colgroups], workspace (grows with N)
    int32_t* counters = nullptr;
    int64_t counters_len = 0;
    float* ws = nullptr;
    size_t ws_bytes = 0;
    // host-API staging buffers
    void* stage_B = nullptr;
    size_t stage_B_bytes = 0;
    float* stage_C = nullptr;
    size_t stage_C_bytes = 0;
    // host-API copy pipeline (dtc_spmm_host with column chunks): copy-in / copy-out streams and
    // per-chunk events, created on first use
    cudaStream_t hstream[2] = {nullptr, nullptr};
    cudaEvent_t hev[2 * 16 + 1] = {};
    // streaming host API (dtc_spmm_host_async): two staging sets, copy streams, per-slot events
    void* as_B[2] = {nullptr, nullptr};
    size_t as_B_bytes[2] = {0, 0};
    float* as_C[2] = {nullptr, nullptr};
    size_t as_C_bytes[2] = {0, 0};
    cudaStream_t as_in = nullptr, as_out = nullptr, as_last = nullptr;
    cudaEvent_t as_ev_in[2] = {}, as_ev_kernel[2] = {}, as_ev_out[2] = {};
    int64_t as_seq = 0;
    // optional row map (row of the condensed matrix -> row of C), from dtc_build_opts_t.row_perm
    int32_t* rowmap = nullptr;
    // launch options and diagnostics
    dtc::Options opt;
    int64_t* trace = nullptr;         // per-CTA timeline buffer (dtc_format_set_trace), caller-owned
    int64_t trace_cap = 0;
    int32_t last_kernel = 0;          // kernel of the last dtc_spmm (1 register gather, 4 padded TMA)
    int64_t last_host_mode = 0;       // last dtc_spmm_host: 2 * chunks + zero-copy C
    // persistent padded-row launch: dynamic unit counters, 2 per column group (self-resetting)
    int32_t* uctr = nullptr;
    int64_t uctr_len = 0;
    dtc::Unit* units_lpt = nullptr;   // units by size, descending (persistent launch)
    int32_t* ufirst = nullptr;        // per-unit first-batch side records (one-CTA-per-unit pad launch)
    // GraphConv (dtc_graphconv): cuBLASLt workspace for the dense (A*H)*W step
    uint8_t* gemm_ws = nullptr;
    size_t gemm_ws_bytes = 0;
};

namespace dtc {

// thread-local last error
void set_error(const char* fmt, ...);
int cuda_fail(cudaError_t e, const char* what, const char* file, int line);

#define DTC_CUDA(call)                                                            \
    do {                                                                          \
        cudaError_t _e = (call);                                                  \
        if (_e != cudaSuccess) return ::dtc::cuda_fail(_e, #call, __FILE__, __LINE__); \
    } while (0)

// device-wide exclusive scan of n int64 values (in != out allowed, in-place
// allowed); out[n] receives the total.  tmp must hold scan_tmp_elems(n).
int64_t scan_tmp_elems(int64_t n);
void exclusive_scan_i64(const int64_t* in, int64_t* out, int64_t n, int64_t* tmp,
                        cudaStream_t s);

inline int elt_size(int32_t dtype) { return dtype == DTC_FP16 ? 2 : 4; }

// Stream-ordered device allocations come from a library-owned memory pool per
// device whose release threshold is "never": freed blocks stay cached, so a
// second build / a growing workspace does not pay the OS map/unmap cost again.
cudaMemPool_t lib_pool();

template <class T>
int dalloc(T** p, size_t count, cudaStream_t s) {
    *p = nullptr;
    if (count == 0) count = 1;
    cudaError_t e = cudaMallocFromPoolAsync(reinterpret_cast<void**>(p), count * sizeof(T), lib_pool(), s);
    if (e != cudaSuccess) {
        cudaGetLastError();
        set_error("device allocation of %zu bytes failed: %s", count * sizeof(T), cudaGetErrorString(e));
        return DTC_ERR_OOM;
    }
    return DTC_OK;
}
template <class T>
void dfree(T*& p, cudaStream_t s) {
    if (p) cudaFreeAsync(reinterpret_cast<void*>(p), s);
    p = nullptr;
}

// small pinned host buffer (per thread) for the build's blocking scalar readbacks
int64_t* pinned_scratch();

int num_sms();

// SpMM kernel launcher (dtc_spmm.cu)
int spmm_launch(dtc_format* h, const void* B, int64_t N, int64_t ldb, float* C, int64_t ldc,
                cudaStream_t s);

// padded-path geometry and measured occupancy for N columns (dtc_spmm.cu), used by the Selector
struct PadGeometry {
    int seg, slices;
    int64_t cta_cols;
};
PadGeometry pad_geometry(int dtype, int64_t N, int slice_bytes);
int pad_occupancy(int dtype, int64_t N, int window_h = 16);

// B200 Selector (dtc_selector.cu): simulate the F4 units of each candidate plan, return the best
int selector_plan(const int32_t* rwo, int64_t W, const dtc_sched_model_t& m, const int32_t* cand, int ncand,
                  int guided_opt, dtc_plan_t* plans, dtc_plan_t* best);
int sched_model(int dtype, int64_t N, dtc_sched_model_t* m, int window_h = 16);

// F0-F2 only (dtc_format.cu): validated RowWindowOffset of 16-row windows, on the host
int window_offsets(const dtc_csr_t* csr, cudaStream_t s, std::vector<int32_t>* rwo_out, int window_h = 16);

// internal build used by the distributed layer: optional row range of the csr
int format_build(const dtc_csr_t* csr, const dtc_build_opts_t* opts, cudaStream_t s,
                 dtc_format** out);

}  // namespace dtc
