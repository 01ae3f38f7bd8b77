// dtc_host.cu -- the end-to-end host-buffer entry point (dtc_spmm_host) and the per-handle
// launch options.  The kernels are dtc_spmm.cu's; nothing here computes.
#include <algorithm>
#include <cstdlib>

#include "dtc_internal.h"

namespace dtc {

// Column chunks for dtc_spmm_host: C(:, cols) depends only on B(:, cols), so the call is pipelined
// over column chunks -- H2D of chunk j+1 runs while chunk j computes and its C chunk goes back
// (PCIe / C2C are full duplex).  Every output element is the same sum in the same order as one
// dtc_spmm over all N columns (the kernels' per-column arithmetic does not depend on N).
// Pitched copies of narrow row pieces run well below the wide-copy rate, and each chunk's kernel
// re-reads the format (A), so chunks keep >= 512 B of a B row, or >= 256 B when the format is
// smaller than B (the kernels are short next to the copies); at most 4 chunks.  Measured on B200,
// dtc_spmm_host e2e (profiles/r01_host_chunks.txt): c2 2 x 256 B +24%, c4 2 x 256 B +27%, c3 2 x 512 B
// +27%, c5 4 x 512 B +58%; c3h (FP16, format 5x B) 2 x 256 B -12%, so it stays unpipelined.
// DTC_OPT_HOST_CHUNKS overrides the count (1 = the unpipelined copy-in, kernel, copy-out sequence).
static double format_bytes(const dtc_format* h, int elt) {
    return (double)h->nnz * (elt + 1) + 36.0 * (double)h->T + 4.0 * (double)h->W;
}

static int host_chunks(const dtc_format* h, int64_t N, int elt, size_t bytes) {
    const int64_t row = N * elt;
    const double b_bytes = (double)std::max<int64_t>(h->K, 1) * row;
    const int64_t wmin = format_bytes(h, elt) < b_bytes ? 256 : 512;
    int64_t c = std::min<int64_t>(4, row / wmin);
    if (bytes < ((size_t)8 << 20)) c = 1;   // small calls: latency, not bandwidth
    if (h->opt.host_chunks > 0) c = h->opt.host_chunks;
    return (int)std::max<int64_t>(1, std::min<int64_t>({c, 16, (N + 31) / 32}));   // widths: multiples of 32 columns
}

// after an error: let every copy already queued against the caller's host buffers finish before
// returning (the buffers must not be touched once the call has returned)
static void drain(dtc_format* h, cudaStream_t s) {
    cudaStreamSynchronize(s);
    for (auto& hs : h->hstream)
        if (hs) cudaStreamSynchronize(hs);
    cudaGetLastError();
}

static int ensure_copy_streams(dtc_format* h) {
    for (auto& hs : h->hstream)
        if (!hs) DTC_CUDA(cudaStreamCreateWithFlags(&hs, cudaStreamNonBlocking));
    for (auto& e : h->hev)
        if (!e) DTC_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    return DTC_OK;
}

static int spmm_host_impl(dtc_format* h, const void* B_host, int64_t N, int64_t ldb, float* C_host, int64_t ldc,
                          cudaStream_t s) {
    const int elt = elt_size(h->dtype);
    const size_t bbytes = (size_t)std::max<int64_t>(h->K, 1) * N * elt;
    const size_t cbytes = (size_t)std::max<int64_t>(h->M, 1) * N * sizeof(float);
    const int nch = host_chunks(h, N, elt, bbytes + cbytes);
    // Zero-copy C: when C_host is pinned and mapped, the kernel stores C straight into host memory
    // (posted PCIe writes spread over the kernel) and the copy-out disappears.  It pays when the
    // kernel is long next to the copies (format larger than B: c3 e2e 12.1 -> 10.1 ms) and costs
    // 1-5% otherwise (c2, c4, c5; profiles/r01_host_zc.txt).  DTC_OPT_HOST_ZERO_COPY overrides.
    float* Czc = nullptr;
    {
        bool zc = format_bytes(h, elt) > (double)bbytes && bbytes + cbytes >= ((size_t)8 << 20);
        if (h->opt.host_zc >= 0) zc = h->opt.host_zc > 0;
        if (zc) {
            cudaPointerAttributes at{};
            if (cudaPointerGetAttributes(&at, C_host) != cudaSuccess) cudaGetLastError();   // unregistered memory
            else if (at.type == cudaMemoryTypeHost && at.devicePointer) Czc = reinterpret_cast<float*>(at.devicePointer);
        }
    }
    h->last_host_mode = (int64_t)nch * 2 + (Czc ? 1 : 0);
    if (bbytes > h->stage_B_bytes) {
        dfree(h->stage_B, s);
        h->stage_B_bytes = 0;
        uint8_t* sb = nullptr;
        int rc = dalloc(&sb, bbytes, s);
        if (rc) return rc;
        h->stage_B = sb;
        h->stage_B_bytes = bbytes;
    }
    if (!Czc && cbytes > h->stage_C_bytes) {   // the zero-copy path needs no device C
        dfree(h->stage_C, s);
        h->stage_C_bytes = 0;
        int rc = dalloc(&h->stage_C, cbytes / sizeof(float), s);
        if (rc) return rc;
        h->stage_C_bytes = cbytes;
    }
    uint8_t* sb = reinterpret_cast<uint8_t*>(h->stage_B);
    if (nch <= 1 && !Czc) {
        if (h->K > 0)
            DTC_CUDA(cudaMemcpy2DAsync(sb, N * elt, B_host, ldb * elt, N * elt, h->K, cudaMemcpyHostToDevice, s));
        int rc = spmm_launch(h, sb, N, N, h->stage_C, N, s);
        if (rc) return rc;
        if (h->M > 0)
            DTC_CUDA(cudaMemcpy2DAsync(C_host, ldc * sizeof(float), h->stage_C, N * sizeof(float), N * sizeof(float),
                                       h->M, cudaMemcpyDeviceToHost, s));
        DTC_CUDA(cudaStreamSynchronize(s));
        return DTC_OK;
    }
    int rc = ensure_copy_streams(h);
    if (rc) return rc;
    cudaStream_t sin = h->hstream[0], sout = h->hstream[1];
    cudaEvent_t* evb = h->hev;         // [nch] chunk j of B resident
    cudaEvent_t* evk = h->hev + 16;    // [nch] chunk j of C computed
    cudaEvent_t evs = h->hev[32];      // start / end fence
    // the copy streams start after everything already queued on s (e.g. staging reallocation)
    DTC_CUDA(cudaEventRecord(evs, s));
    DTC_CUDA(cudaStreamWaitEvent(sin, evs, 0));
    DTC_CUDA(cudaStreamWaitEvent(sout, evs, 0));
    // chunk widths: multiples of 32 columns, the remainder spread over the first chunks
    const int64_t units32 = (N + 31) / 32;
    int64_t c0 = 0;
    for (int j = 0; j < nch; ++j) {
        const int64_t u = units32 / nch + (j < units32 % nch ? 1 : 0);
        const int64_t nc = std::min<int64_t>(N - c0, u * 32);
        uint8_t* bj = sb + (size_t)h->K * c0 * elt;                 // K x nc, ldb = nc
        if (h->K > 0)
            DTC_CUDA(cudaMemcpy2DAsync(bj, nc * elt, reinterpret_cast<const uint8_t*>(B_host) + c0 * elt, ldb * elt,
                                       nc * elt, h->K, cudaMemcpyHostToDevice, sin));
        DTC_CUDA(cudaEventRecord(evb[j], sin));
        DTC_CUDA(cudaStreamWaitEvent(s, evb[j], 0));
        if (Czc) {   // the kernel writes the chunk's C columns straight into the mapped host buffer
            rc = spmm_launch(h, bj, nc, nc, Czc + c0, ldc, s);
            if (rc) return rc;
        } else {
            float* cj = h->stage_C + (size_t)h->M * c0;                // M x nc, ldc = nc
            rc = spmm_launch(h, bj, nc, nc, cj, nc, s);
            if (rc) return rc;
            DTC_CUDA(cudaEventRecord(evk[j], s));
            DTC_CUDA(cudaStreamWaitEvent(sout, evk[j], 0));
            if (h->M > 0)
                DTC_CUDA(cudaMemcpy2DAsync(C_host + c0, ldc * sizeof(float), cj, nc * sizeof(float),
                                           nc * sizeof(float), h->M, cudaMemcpyDeviceToHost, sout));
        }
        c0 += nc;
    }
    if (!Czc) {
        DTC_CUDA(cudaEventRecord(evs, sout));
        DTC_CUDA(cudaStreamWaitEvent(s, evs, 0));
    }
    DTC_CUDA(cudaStreamSynchronize(s));
    return DTC_OK;
}

}  // namespace dtc

using namespace dtc;

extern "C" int dtc_spmm_host(dtc_handle_t h, const void* B_host, int64_t N, int64_t ldb, float* C_host,
                             int64_t ldc, void* stream) {
    if (!h || !C_host || (!B_host && h->K > 0)) { set_error("null argument"); return DTC_ERR_INVALID; }
    if (N < 1 || ldb < N || ldc < N) { set_error("bad N/ldb/ldc"); return DTC_ERR_INVALID; }
    int prev = -1;
    if (cudaGetDevice(&prev) != cudaSuccess) { cudaGetLastError(); set_error("no CUDA device"); return DTC_ERR_CUDA; }
    if (prev != h->device && cudaSetDevice(h->device) != cudaSuccess) {
        cudaGetLastError();
        set_error("cannot select the handle's device %d", h->device);
        return DTC_ERR_CUDA;
    }
    cudaStream_t s = (cudaStream_t)stream;
    const int rc = spmm_host_impl(h, B_host, N, ldb, C_host, ldc, s);
    if (rc != DTC_OK) drain(h, s);
    if (prev != h->device) cudaSetDevice(prev);
    return rc;
}

// ------------------------------------------------------------ streaming host API
// Call j uses staging slot j & 1: its copy-in waits (on the device) for call j-2's kernel to have
// read that slot's B, its kernel for call j-2's copy-out to have drained that slot's C; nothing
// waits on the host.  So consecutive calls overlap: copy-in of j+1 || kernel of j || copy-out of
// j-1 (PCIe is full duplex).  Zero-copy C (pinned mapped C_host, format larger than B) as in
// dtc_spmm_host.  Every call computes exactly what dtc_spmm computes.
static int spmm_host_async_impl(dtc_format* h, const void* B_host, int64_t N, int64_t ldb, float* C_host, int64_t ldc,
                                cudaStream_t s) {
    const int elt = elt_size(h->dtype);
    const size_t bbytes = (size_t)std::max<int64_t>(h->K, 1) * N * elt;
    const size_t cbytes = (size_t)std::max<int64_t>(h->M, 1) * N * sizeof(float);
    const int slot = (int)(h->as_seq & 1);
    float* Czc = nullptr;
    {
        bool zc = format_bytes(h, elt) > (double)bbytes && bbytes + cbytes >= ((size_t)8 << 20);
        if (h->opt.host_zc >= 0) zc = h->opt.host_zc > 0;
        if (zc) {
            cudaPointerAttributes at{};
            if (cudaPointerGetAttributes(&at, C_host) != cudaSuccess) cudaGetLastError();
            else if (at.type == cudaMemoryTypeHost && at.devicePointer) Czc = reinterpret_cast<float*>(at.devicePointer);
        }
    }
    h->last_host_mode = 2 + (Czc ? 1 : 0);
    if (!h->as_in) DTC_CUDA(cudaStreamCreateWithFlags(&h->as_in, cudaStreamNonBlocking));
    if (!h->as_out) DTC_CUDA(cudaStreamCreateWithFlags(&h->as_out, cudaStreamNonBlocking));
    for (int k = 0; k < 2; ++k) {
        if (!h->as_ev_in[k]) DTC_CUDA(cudaEventCreateWithFlags(&h->as_ev_in[k], cudaEventDisableTiming));
        if (!h->as_ev_kernel[k]) DTC_CUDA(cudaEventCreateWithFlags(&h->as_ev_kernel[k], cudaEventDisableTiming));
        if (!h->as_ev_out[k]) DTC_CUDA(cudaEventCreateWithFlags(&h->as_ev_out[k], cudaEventDisableTiming));
    }
    // (re)size this slot's staging: freed in stream order after the slot's previous kernel / copy-out
    const bool realloc = bbytes > h->as_B_bytes[slot] || (!Czc && cbytes > h->as_C_bytes[slot]);
    if (realloc) {
        DTC_CUDA(cudaStreamWaitEvent(s, h->as_ev_kernel[slot], 0));
        DTC_CUDA(cudaStreamWaitEvent(s, h->as_ev_out[slot], 0));
    }
    if (bbytes > h->as_B_bytes[slot]) {
        dfree(h->as_B[slot], s);
        h->as_B_bytes[slot] = 0;
        uint8_t* b = nullptr;
        int rc = dalloc(&b, bbytes, s);
        if (rc) return rc;
        h->as_B[slot] = b;
        h->as_B_bytes[slot] = bbytes;
    }
    if (!Czc && cbytes > h->as_C_bytes[slot]) {
        dfree(h->as_C[slot], s);
        h->as_C_bytes[slot] = 0;
        int rc = dalloc(&h->as_C[slot], cbytes / sizeof(float), s);
        if (rc) return rc;
        h->as_C_bytes[slot] = cbytes;
    }
    // copy-in after call j-2's kernel (it read this slot's B) -- and, when this call (re)allocated the
    // slot, after the stream-ordered allocation on s; otherwise NOT after s's queue, so the copy-in
    // of call j+1 overlaps the kernel of call j
    if (realloc) {
        DTC_CUDA(cudaEventRecord(h->as_ev_in[slot], s));
        DTC_CUDA(cudaStreamWaitEvent(h->as_in, h->as_ev_in[slot], 0));
    }
    DTC_CUDA(cudaStreamWaitEvent(h->as_in, h->as_ev_kernel[slot], 0));
    if (h->K > 0)
        DTC_CUDA(cudaMemcpy2DAsync(h->as_B[slot], N * elt, B_host, ldb * elt, N * elt, h->K, cudaMemcpyHostToDevice,
                                   h->as_in));
    DTC_CUDA(cudaEventRecord(h->as_ev_in[slot], h->as_in));
    DTC_CUDA(cudaStreamWaitEvent(s, h->as_ev_in[slot], 0));
    if (Czc) {
        int rc = spmm_launch(h, h->as_B[slot], N, N, Czc, ldc, s);
        if (rc) return rc;
        DTC_CUDA(cudaEventRecord(h->as_ev_kernel[slot], s));
        DTC_CUDA(cudaEventRecord(h->as_ev_out[slot], s));
    } else {
        DTC_CUDA(cudaStreamWaitEvent(s, h->as_ev_out[slot], 0));   // call j-2's copy-out drained this C slot
        int rc = spmm_launch(h, h->as_B[slot], N, N, h->as_C[slot], N, s);
        if (rc) return rc;
        DTC_CUDA(cudaEventRecord(h->as_ev_kernel[slot], s));
        DTC_CUDA(cudaStreamWaitEvent(h->as_out, h->as_ev_kernel[slot], 0));
        if (h->M > 0)
            DTC_CUDA(cudaMemcpy2DAsync(C_host, ldc * sizeof(float), h->as_C[slot], N * sizeof(float), N * sizeof(float),
                                       h->M, cudaMemcpyDeviceToHost, h->as_out));
        DTC_CUDA(cudaEventRecord(h->as_ev_out[slot], h->as_out));
    }
    h->as_last = s;
    ++h->as_seq;
    return DTC_OK;
}

extern "C" int dtc_spmm_host_async(dtc_handle_t h, const void* B_host, int64_t N, int64_t ldb, float* C_host,
                                   int64_t ldc, void* stream) {
    if (!h || !C_host || (!B_host && h->K > 0)) { set_error("null argument"); return DTC_ERR_INVALID; }
    if (N < 1 || ldb < N || ldc < N) { set_error("bad N/ldb/ldc"); return DTC_ERR_INVALID; }
    int prev = -1;
    if (cudaGetDevice(&prev) != cudaSuccess) { cudaGetLastError(); set_error("no CUDA device"); return DTC_ERR_CUDA; }
    if (prev != h->device && cudaSetDevice(h->device) != cudaSuccess) {
        cudaGetLastError();
        set_error("cannot select the handle's device %d", h->device);
        return DTC_ERR_CUDA;
    }
    const int rc = spmm_host_async_impl(h, B_host, N, ldb, C_host, ldc, (cudaStream_t)stream);
    if (prev != h->device) cudaSetDevice(prev);
    return rc;
}

extern "C" int dtc_spmm_host_wait(dtc_handle_t h) {
    if (!h) { set_error("null handle"); return DTC_ERR_INVALID; }
    int prev = -1;
    if (cudaGetDevice(&prev) != cudaSuccess) { cudaGetLastError(); set_error("no CUDA device"); return DTC_ERR_CUDA; }
    if (prev != h->device) cudaSetDevice(h->device);
    cudaError_t e = cudaSuccess;
    auto sync = [&](cudaStream_t st) {
        const cudaError_t e2 = cudaStreamSynchronize(st);
        if (e == cudaSuccess) e = e2;
    };
    if (h->as_in) sync(h->as_in);
    if (h->as_seq > 0) sync(h->as_last);   // the compute stream of the last call (may be the legacy stream)
    if (h->as_out) sync(h->as_out);
    if (prev != h->device) cudaSetDevice(prev);
    if (e != cudaSuccess) return cuda_fail(e, "dtc_spmm_host_wait", __FILE__, __LINE__);
    return DTC_OK;
}

extern "C" int dtc_format_set_option(dtc_handle_t h, int32_t option, int64_t value) {
    if (!h) { set_error("null handle"); return DTC_ERR_INVALID; }
    auto bad = [&]() {
        set_error("option %d: value %lld out of range", (int)option, (long long)value);
        return (int)DTC_ERR_INVALID;
    };
    switch (option) {
        case DTC_OPT_KERNEL:
            if (value != 0 && value != 1 && value != 4) return bad();
            h->opt.kernel = (int32_t)value;
            return DTC_OK;
        case DTC_OPT_PERSISTENT:
            if (value != 0 && value != 1) return bad();
            h->opt.persistent = (int32_t)value;
            return DTC_OK;
        case DTC_OPT_FIRST_RECORDS:
            if (value != 0 && value != 1) return bad();
            h->opt.first_records = (int32_t)value;
            return DTC_OK;
        case DTC_OPT_HOST_CHUNKS:
            if (value < 0 || value > 16) return bad();
            h->opt.host_chunks = (int32_t)value;
            return DTC_OK;
        case DTC_OPT_HOST_ZERO_COPY:
            if (value < -1 || value > 1) return bad();
            h->opt.host_zc = (int32_t)value;
            return DTC_OK;
        case DTC_OPT_SLICE_BYTES:
            if (value != 0 && value != 512 && value != 1024) return bad();
            h->opt.slice_bytes = (int32_t)value;
            return DTC_OK;
        default:
            set_error("option %d is unknown or read-only", (int)option);
            return DTC_ERR_INVALID;
    }
}

extern "C" int dtc_format_get_option(dtc_handle_t h, int32_t option, int64_t* value) {
    if (!h || !value) { set_error("null argument"); return DTC_ERR_INVALID; }
    switch (option) {
        case DTC_OPT_KERNEL: *value = h->opt.kernel; return DTC_OK;
        case DTC_OPT_PERSISTENT: *value = h->opt.persistent; return DTC_OK;
        case DTC_OPT_FIRST_RECORDS: *value = h->opt.first_records; return DTC_OK;
        case DTC_OPT_HOST_CHUNKS: *value = h->opt.host_chunks; return DTC_OK;
        case DTC_OPT_HOST_ZERO_COPY: *value = h->opt.host_zc; return DTC_OK;
        case DTC_OPT_SLICE_BYTES: *value = h->opt.slice_bytes; return DTC_OK;
        case DTC_OPT_LAST_KERNEL: *value = h->last_kernel; return DTC_OK;
        case DTC_OPT_LAST_HOST_MODE: *value = h->last_host_mode; return DTC_OK;
        case DTC_OPT_GUIDED: *value = h->guided; return DTC_OK;
        case DTC_OPT_PLAN_MAKESPAN_NS: *value = (int64_t)(h->plan_makespan_ns + 0.5); return DTC_OK;
        default: set_error("option %d is unknown", (int)option); return DTC_ERR_INVALID;
    }
}

extern "C" int dtc_format_set_trace(dtc_handle_t h, void* dev_buf, int64_t capacity_ctas) {
    if (!h || capacity_ctas < 0 || (capacity_ctas > 0 && !dev_buf)) { set_error("bad trace buffer"); return DTC_ERR_INVALID; }
    h->trace = capacity_ctas ? reinterpret_cast<int64_t*>(dev_buf) : nullptr;
    h->trace_cap = capacity_ctas;
    return DTC_OK;
}
