// dtc_dist.cu -- multi-GPU row-window data parallelism (north_star; the paper is
// single-GPU, its parallelism is row windows across SMs).
//
// One process per GPU.  Windows are split into contiguous ranges balanced by
// TC-block count (prefix of RowWindowOffset, from F0-F2 only); each rank condenses
// only its CSR row slice.  The single exchange is B: every rank needs all of it
// because the columns of A are arbitrary, so the root broadcasts it with NCCL over
// NVLink/NVSwitch -- in column chunks, pipelined with the kernel: C(:, cols)
// depends only on B(:, cols), so chunk j+1 crosses NVLink (comm stream) while
// chunk j computes (compute stream).  C can be all-gathered (each owner
// broadcasts its rows, grouped), otherwise each rank keeps its own rows.
#include <nccl.h>

#include <algorithm>
#include <new>
#include <vector>

#include "dtc_internal.h"

constexpr int kMaxDistChunks = 8;

struct dtc_dist {
    int rank = 0, world = 1;
    int64_t M = 0, K = 0;
    int32_t dtype = 0;
    std::vector<int64_t> row_begin;  // [world+1]
    dtc_format* local = nullptr;
    int32_t* local_rowptr = nullptr;
    ncclComm_t comm = nullptr;
    // chunked broadcast: library-owned chunk-major copy of B, comm stream, per-chunk events
    uint8_t* stage = nullptr;
    size_t stage_bytes = 0;
    cudaStream_t comm_stream = nullptr;
    cudaEvent_t ev_in = nullptr, ev_out = nullptr;
    cudaEvent_t ev_chunk[kMaxDistChunks] = {};
    int32_t chunks_opt = 0;          // 0 = auto
};

namespace dtc {

static int nccl_fail(ncclResult_t r, const char* what) {
    set_error("%s failed: %s", what, ncclGetErrorString(r));
    return DTC_ERR_NCCL;
}
#define DTC_NCCL(call)                                              \
    do {                                                            \
        ncclResult_t _r = (call);                                   \
        if (_r != ncclSuccess) return ::dtc::nccl_fail(_r, #call);  \
    } while (0)

// pack B(:, columns [off, off + w)) (row pitch ldb bytes) into a contiguous K x w block: one pass at
// HBM rate (a pitched cudaMemcpy2D of narrow rows runs far below it); V = bytes per access
template <class V>
__global__ void k_pack_cols(const uint8_t* __restrict__ B, int64_t ldb, int64_t off, int64_t w, int64_t K,
                            uint8_t* __restrict__ dst) {
    const int64_t per_row = w / (int64_t)sizeof(V), n = per_row * K;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = i / per_row, k = i - r * per_row;
        reinterpret_cast<V*>(dst + r * w)[k] = *reinterpret_cast<const V*>(B + r * ldb + off + k * (int64_t)sizeof(V));
    }
}

static cudaError_t pack_cols(const void* B, int64_t ldb, int64_t off, int64_t w, int64_t K, void* dst, cudaStream_t s) {
    const uintptr_t a = (uintptr_t)B | (uintptr_t)dst | (uintptr_t)ldb | (uintptr_t)off | (uintptr_t)w;
    const unsigned grid = 148 * 8;
    if (a % 16 == 0)
        k_pack_cols<uint4><<<grid, 256, 0, s>>>((const uint8_t*)B, ldb, off, w, K, (uint8_t*)dst);
    else if (a % 4 == 0)
        k_pack_cols<uint32_t><<<grid, 256, 0, s>>>((const uint8_t*)B, ldb, off, w, K, (uint8_t*)dst);
    else
        k_pack_cols<uint8_t><<<grid, 256, 0, s>>>((const uint8_t*)B, ldb, off, w, K, (uint8_t*)dst);
    return cudaGetLastError();
}

__global__ void k_rebase(const int32_t* __restrict__ in, int32_t* __restrict__ out, int64_t n, int32_t base) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = in[i] - base;
}

}  // namespace dtc

using namespace dtc;

extern "C" int dtc_partition_windows(const int32_t* rwo, int64_t W, int32_t world, int64_t* w_begin) {
    if (!rwo || !w_begin || W < 0 || world < 1) { set_error("bad partition arguments"); return DTC_ERR_INVALID; }
    const int64_t T = rwo[W];
    w_begin[0] = 0;
    int64_t w = 0;
    for (int r = 1; r < world; ++r) {
        // smallest w with rwo[w] >= r*T/world (ceil), never before the previous cut
        const int64_t target = (T * r + world - 1) / world;
        while (w < W && rwo[w] < target) ++w;
        w_begin[r] = w;
    }
    w_begin[world] = W;
    return DTC_OK;
}

extern "C" int dtc_nccl_unique_id(void* out128) {
    if (!out128) { set_error("null output"); return DTC_ERR_INVALID; }
    ncclUniqueId id;
    DTC_NCCL(ncclGetUniqueId(&id));
    static_assert(sizeof(ncclUniqueId) == 128, "NCCL unique id is 128 bytes");
    memcpy(out128, &id, sizeof(id));
    return DTC_OK;
}

extern "C" int dtc_dist_create(const dtc_csr_t* csr, int32_t rank, int32_t world, const void* nccl_id, void* stream,
                               dtc_dist_t* out) {
    if (!out) { set_error("out is NULL"); return DTC_ERR_INVALID; }
    *out = nullptr;
    if (!csr || world < 1 || rank < 0 || rank >= world) { set_error("bad rank/world"); return DTC_ERR_INVALID; }
    cudaStream_t s = (cudaStream_t)stream;
    // 1. window partition from the full matrix's RowWindowOffset (F0-F2 only: counts, no format)
    std::vector<int32_t> rwo;
    int rc = window_offsets(csr, s, &rwo);
    if (rc) return rc;
    cudaError_t e = cudaSuccess;
    std::vector<int64_t> wb(world + 1);
    dtc_partition_windows(rwo.data(), (int64_t)rwo.size() - 1, world, wb.data());
    dtc_dist* d = new (std::nothrow) dtc_dist();
    if (!d) { set_error("host OOM"); return DTC_ERR_OOM; }
    d->rank = rank; d->world = world; d->M = csr->M; d->K = csr->K; d->dtype = csr->dtype;
    d->row_begin.resize(world + 1);
    for (int r = 0; r <= world; ++r) d->row_begin[r] = std::min<int64_t>(wb[r] * kWindow, csr->M);
    // 2. local CSR slice (rows [r0, r1)), rowptr rebased to 0
    const int64_t r0 = d->row_begin[rank], r1 = d->row_begin[rank + 1];
    int32_t base = 0, endp = 0;
    if (csr->M > 0) {
        e = cudaMemcpy(&base, csr->rowptr + r0, sizeof(int32_t), cudaMemcpyDeviceToHost);
        if (e == cudaSuccess) e = cudaMemcpy(&endp, csr->rowptr + r1, sizeof(int32_t), cudaMemcpyDeviceToHost);
        if (e != cudaSuccess) { delete d; return cuda_fail(e, "rowptr readback", __FILE__, __LINE__); }
    }
    rc = dalloc(&d->local_rowptr, r1 - r0 + 1, s);
    if (rc) { delete d; return rc; }
    k_rebase<<<64, 256, 0, s>>>(csr->rowptr + r0, d->local_rowptr, r1 - r0 + 1, base);
    dtc_csr_t lc;
    lc.M = r1 - r0; lc.K = csr->K; lc.nnz = endp - base;
    lc.rowptr = d->local_rowptr;
    lc.colidx = csr->colidx + base;
    lc.vals = (const char*)csr->vals + (int64_t)base * elt_size(csr->dtype);
    lc.dtype = csr->dtype;
    rc = format_build(&lc, nullptr, s, &d->local);
    if (rc) { dfree(d->local_rowptr, s); cudaStreamSynchronize(s); delete d; return rc; }
    // 3. communicator
    if (nccl_id) {   // a 1-rank communicator is valid too (exercises the NCCL path on one GPU)
        ncclUniqueId id;
        memcpy(&id, nccl_id, sizeof(id));
        ncclResult_t nr = ncclCommInitRank(&d->comm, world, id, rank);
        if (nr != ncclSuccess) {
            dtc_format_destroy(d->local);
            dfree(d->local_rowptr, s);
            cudaStreamSynchronize(s);
            delete d;
            return nccl_fail(nr, "ncclCommInitRank");
        }
    }
    *out = d;
    return DTC_OK;
}

extern "C" int dtc_dist_query(dtc_dist_t d, int64_t* row_begin, int64_t* row_end, dtc_handle_t* local) {
    if (!d) { set_error("null dist"); return DTC_ERR_INVALID; }
    if (row_begin) *row_begin = d->row_begin[d->rank];
    if (row_end) *row_end = d->row_begin[d->rank + 1];
    if (local) *local = d->local;
    return DTC_OK;
}

// Column chunks of the pipelined broadcast: widths are multiples of 32 columns, each chunk >= 128 KB
// of B per rank (smaller NCCL broadcasts are latency bound), at most kMaxDistChunks.
extern "C" int dtc_dist_chunks(int64_t K, int64_t N, int32_t elt, int32_t max_chunks, int64_t* col_begin) {
    if (K < 0 || N < 1 || (elt != 2 && elt != 4) || max_chunks < 0 || !col_begin) {
        set_error("bad dist_chunks arguments");
        return DTC_ERR_INVALID;
    }
    const int64_t units32 = (N + 31) / 32;
    int64_t c = max_chunks > 0 ? max_chunks : 4;
    c = std::min<int64_t>(c, kMaxDistChunks);
    c = std::min<int64_t>(c, units32);
    while (c > 1 && K * (N / c) * elt < (int64_t(128) << 10)) --c;
    c = std::max<int64_t>(c, 1);
    int64_t c0 = 0;
    for (int64_t j = 0; j < c; ++j) {
        col_begin[j] = c0;
        const int64_t u = units32 / c + (j < units32 % c ? 1 : 0);
        c0 = std::min<int64_t>(N, c0 + u * 32);
    }
    col_begin[c] = N;
    return (int)c;   // number of chunks (>= 1)
}

extern "C" int dtc_spmm_dist(dtc_dist_t d, void* B, int32_t root, int64_t N, float* C, int32_t gather_c,
                             void* stream) {
    if (!d || !C || N < 1 || root < 0 || root >= d->world) { set_error("bad dist arguments"); return DTC_ERR_INVALID; }
    if (d->world > 1 && !d->comm) { set_error("no communicator (created with nccl_id == NULL)"); return DTC_ERR_INVALID; }
    if (d->rank == root && !B && d->K > 0) { set_error("B is NULL on the root"); return DTC_ERR_INVALID; }
    cudaStream_t s = (cudaStream_t)stream;
    const int64_t r0 = d->row_begin[d->rank];
    float* Cl = gather_c ? C + r0 * N : C;
    if (!d->comm) {   // communicator-less shard: B is resident, plain local SpMM
        if (!B && d->K > 0) { set_error("B is NULL"); return DTC_ERR_INVALID; }
        return spmm_launch(d->local, B, N, N, Cl, N, s);
    }
    const int elt = elt_size(d->dtype);
    const ncclDataType_t bt = d->dtype == DTC_FP16 ? ncclHalf : ncclFloat;
    int64_t cb[kMaxDistChunks + 1];
    const int nch = dtc_dist_chunks(d->K, N, elt, d->chunks_opt, cb);
    if (nch < 1) return nch;
    // library-owned chunk-major B: chunk j is a contiguous K x n_j block at offset K * cb[j] * elt
    const size_t need = (size_t)std::max<int64_t>(d->K, 1) * N * elt;
    if (need > d->stage_bytes) {
        dfree(d->stage, s);
        d->stage_bytes = 0;
        int rc = dalloc(&d->stage, need, s);
        if (rc) return rc;
        d->stage_bytes = need;
    }
    if (!d->comm_stream) DTC_CUDA(cudaStreamCreateWithFlags(&d->comm_stream, cudaStreamNonBlocking));
    if (!d->ev_in) DTC_CUDA(cudaEventCreateWithFlags(&d->ev_in, cudaEventDisableTiming));
    if (!d->ev_out) DTC_CUDA(cudaEventCreateWithFlags(&d->ev_out, cudaEventDisableTiming));
    for (auto& e : d->ev_chunk)
        if (!e) DTC_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    cudaStream_t cs = d->comm_stream;
    DTC_CUDA(cudaEventRecord(d->ev_in, s));           // B (root) and the staging buffer are ready after s's work
    DTC_CUDA(cudaStreamWaitEvent(cs, d->ev_in, 0));
    for (int j = 0; j < nch; ++j) {
        const int64_t nc = cb[j + 1] - cb[j];
        uint8_t* bj = d->stage + (size_t)d->K * cb[j] * elt;
        if (d->K > 0) {
            if (d->rank == root)   // pack the chunk's columns (strided) into the contiguous chunk buffer
                DTC_CUDA(pack_cols(B, N * elt, cb[j] * elt, nc * elt, d->K, bj, cs));
            DTC_NCCL(ncclBroadcast(bj, bj, (size_t)(d->K * nc), bt, root, d->comm, cs));
        }
        DTC_CUDA(cudaEventRecord(d->ev_chunk[j], cs));
        DTC_CUDA(cudaStreamWaitEvent(s, d->ev_chunk[j], 0));
        int rc = spmm_launch(d->local, bj, nc, nc, Cl + cb[j], N, s);   // C columns [cb[j], cb[j+1]), ldc = N
        if (rc) return rc;
    }
    // the next call may overwrite the staging buffer only after this call's kernels read it
    DTC_CUDA(cudaEventRecord(d->ev_out, s));
    DTC_CUDA(cudaStreamWaitEvent(cs, d->ev_out, 0));
    if (gather_c) {
        DTC_NCCL(ncclGroupStart());
        for (int r = 0; r < d->world; ++r) {
            const int64_t a = d->row_begin[r], b = d->row_begin[r + 1];
            if (b > a) {
                float* p = C + a * N;
                DTC_NCCL(ncclBroadcast(p, p, (size_t)((b - a) * N), ncclFloat, r, d->comm, s));
            }
        }
        DTC_NCCL(ncclGroupEnd());
    }
    return DTC_OK;
}

extern "C" int dtc_dist_set_chunks(dtc_dist_t d, int32_t chunks) {
    if (!d || chunks < 0 || chunks > kMaxDistChunks) { set_error("chunks must be 0 (auto) .. %d", kMaxDistChunks); return DTC_ERR_INVALID; }
    d->chunks_opt = chunks;
    return DTC_OK;
}

extern "C" void dtc_dist_destroy(dtc_dist_t d) {
    if (!d) return;
    if (d->comm_stream) cudaStreamSynchronize(d->comm_stream);
    if (d->comm) ncclCommDestroy(d->comm);
    if (d->stage) { dfree(d->stage, 0); cudaDeviceSynchronize(); }
    for (auto& e : d->ev_chunk)
        if (e) cudaEventDestroy(e);
    if (d->ev_in) cudaEventDestroy(d->ev_in);
    if (d->ev_out) cudaEventDestroy(d->ev_out);
    if (d->comm_stream) cudaStreamDestroy(d->comm_stream);
    dtc_format_destroy(d->local);
    if (d->local_rowptr) { dfree(d->local_rowptr, 0); cudaDeviceSynchronize(); }
    delete d;
}
