// dtc_util.cu -- error reporting, status strings and the device-wide scan used by
// the format builder (F2, F3, F4).
#include <cstdarg>
#include <cstring>
#include <mutex>

#include "dtc_internal.h"

namespace dtc {

static thread_local char g_err[1024] = "";

void set_error(const char* fmt, ...) {
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof(g_err), fmt, ap);
    va_end(ap);
}

int cuda_fail(cudaError_t e, const char* what, const char* file, int line) {
    cudaGetLastError();  // clear sticky-less errors
    set_error("%s failed: %s (%s:%d)", what, cudaGetErrorString(e), file, line);
    return e == cudaErrorMemoryAllocation ? DTC_ERR_OOM : DTC_ERR_CUDA;
}

cudaMemPool_t lib_pool() {
    static cudaMemPool_t pools[64] = {};
    static std::mutex mu;
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= 64) dev = 0;
    std::lock_guard<std::mutex> lock(mu);
    if (!pools[dev]) {
        cudaMemPoolProps props = {};
        props.allocType = cudaMemAllocationTypePinned;
        props.location.type = cudaMemLocationTypeDevice;
        props.location.id = dev;
        cudaMemPool_t p = nullptr;
        if (cudaMemPoolCreate(&p, &props) != cudaSuccess) {
            cudaGetLastError();
            cudaDeviceGetDefaultMemPool(&p, dev);
        }
        uint64_t keep = ~uint64_t(0);
        cudaMemPoolSetAttribute(p, cudaMemPoolAttrReleaseThreshold, &keep);
        pools[dev] = p;
    }
    return pools[dev];
}

int64_t* pinned_scratch() {
    static thread_local int64_t* buf = nullptr;
    if (!buf && cudaMallocHost(reinterpret_cast<void**>(&buf), 64 * sizeof(int64_t)) != cudaSuccess) {
        cudaGetLastError();
        buf = nullptr;
    }
    return buf;
}

int num_sms() {
    int dev = 0, n = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return 148;
    if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) return 148;
    return n;
}

// ------------------------------------------------------------------ scan
constexpr int kScanThreads = 256;
constexpr int kScanItems = 8;
constexpr int kScanTile = kScanThreads * kScanItems;

__device__ __forceinline__ int64_t block_exclusive_scan(int64_t v, int64_t* total) {
    __shared__ int64_t warp_sums[kScanThreads / 32];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    int64_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        int64_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) warp_sums[warp] = x;
    __syncthreads();
    if (warp == 0) {
        int64_t w = lane < kScanThreads / 32 ? warp_sums[lane] : 0;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            int64_t y = __shfl_up_sync(0xffffffffu, w, o);
            if (lane >= o) w += y;
        }
        if (lane < kScanThreads / 32) warp_sums[lane] = w;  // inclusive
    }
    __syncthreads();
    int64_t base = warp > 0 ? warp_sums[warp - 1] : 0;
    *total = warp_sums[kScanThreads / 32 - 1];
    __syncthreads();
    return base + x - v;  // exclusive
}

__global__ void scan_tile_sums(const int64_t* __restrict__ in, int64_t n, int64_t* __restrict__ sums) {
    int64_t base = (int64_t)blockIdx.x * kScanTile + (int64_t)threadIdx.x * kScanItems;
    int64_t s = 0;
#pragma unroll
    for (int i = 0; i < kScanItems; ++i)
        if (base + i < n) s += in[base + i];
    int64_t tot;
    block_exclusive_scan(s, &tot);
    if (threadIdx.x == 0) sums[blockIdx.x] = tot;
}

__global__ void scan_tiles(const int64_t* in, int64_t* out, int64_t n, const int64_t* offsets) {
    int64_t base = (int64_t)blockIdx.x * kScanTile + (int64_t)threadIdx.x * kScanItems;
    int64_t v[kScanItems];
    int64_t s = 0;
#pragma unroll
    for (int i = 0; i < kScanItems; ++i) {
        v[i] = (base + i < n) ? in[base + i] : 0;
        s += v[i];
    }
    int64_t tot;
    int64_t ex = block_exclusive_scan(s, &tot);  // all reads of the tile happen before this barrier
    int64_t off = offsets ? offsets[blockIdx.x] : 0;
    int64_t run = off + ex;
#pragma unroll
    for (int i = 0; i < kScanItems; ++i) {
        if (base + i < n) out[base + i] = run;
        run += v[i];
    }
    if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0) out[n] = off + tot;
}

int64_t scan_tmp_elems(int64_t n) {
    int64_t nb = (n + kScanTile - 1) / kScanTile;
    if (nb <= 1) return 2;
    return nb + 1 + scan_tmp_elems(nb);
}

void exclusive_scan_i64(const int64_t* in, int64_t* out, int64_t n, int64_t* tmp, cudaStream_t s) {
    int64_t nb = (n + kScanTile - 1) / kScanTile;
    if (nb <= 1) {
        scan_tiles<<<1, kScanThreads, 0, s>>>(in, out, n, nullptr);
        return;
    }
    int64_t* sums = tmp;            // [nb + 1]
    int64_t* rest = tmp + nb + 1;
    scan_tile_sums<<<(unsigned)nb, kScanThreads, 0, s>>>(in, n, sums);
    exclusive_scan_i64(sums, sums, nb, rest, s);
    scan_tiles<<<(unsigned)nb, kScanThreads, 0, s>>>(in, out, n, sums);
}

}  // namespace dtc

extern "C" const char* dtc_status_string(int status) {
    switch (status) {
        case DTC_OK: return "DTC_OK";
        case DTC_ERR_INVALID: return "DTC_ERR_INVALID";
        case DTC_ERR_UNSORTED: return "DTC_ERR_UNSORTED";
        case DTC_ERR_DUPLICATE: return "DTC_ERR_DUPLICATE";
        case DTC_ERR_RANGE: return "DTC_ERR_RANGE";
        case DTC_ERR_OOM: return "DTC_ERR_OOM";
        case DTC_ERR_CUDA: return "DTC_ERR_CUDA";
        case DTC_ERR_NCCL: return "DTC_ERR_NCCL";
        case DTC_ERR_UNSUPPORTED: return "DTC_ERR_UNSUPPORTED";
        default: return "DTC_ERR_UNKNOWN";
    }
}

extern "C" const char* dtc_last_error(void) { return dtc::g_err; }

extern "C" const char* dtc_version(void) {
    return "libdtc 0.1 (sm_100a; ME-TCF builder + mma.sync SpMM + NCCL dist)";
}
