// gather_bw2.cu -- microbenchmark (not product code): per-SM throughput of random B-row gathers into
// shared memory on sm_100a, by the two TMA paths the SpMM kernel could use for S2:
//   mode 0: cp.async.bulk.tensor.2d tile::gather4 -- 4 rows x row_bytes per op (the product's path)
//   mode 1: cp.async.bulk (1D)                    -- 1 row x row_bytes per op
// One producer warp per CTA issues `ops` ops per stage (lanes 0..ops-1), R stages, one consumer warp
// releases stages.  Rows are pseudo-random over a K x row_bytes matrix (L2- or DRAM-resident).
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>

__device__ __forceinline__ uint32_t hash32(uint32_t x) {
    x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16;
    return x;
}
__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void k_gather(const __grid_constant__ CUtensorMap map, const uint8_t* __restrict__ B, int K, int row_bytes,
                         int mode, int ops, int R, int iters, int* sink) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ __align__(8) uint64_t full[16], empty[16];
    uint8_t* ring = (uint8_t*)(((uintptr_t)sm + 127) & ~(uintptr_t)127);
    const int rows_per_op = mode == 0 ? 4 : 1;
    const int pitch = row_bytes + 16;                       // padded rows, as in k_spmm_pad
    const int op_bytes = rows_per_op * pitch;
    const int stage_bytes = ops * ((op_bytes + 127) / 128 * 128);
    const int tx = ops * rows_per_op * (mode == 0 ? pitch : row_bytes);
    if (threadIdx.x == 0) {
        for (int i = 0; i < R; ++i) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&full[i])));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&empty[i])));
        }
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    uint32_t seed = blockIdx.x * 7919u;
    if (warp == 0) {
        for (int i = 0; i < iters; ++i) {
            const int s = i % R;
            if (i >= R) {
                uint32_t par = ((i / R) - 1) & 1;
                asm volatile("{\n.reg .pred p;\nW1: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W1;\n}\n" ::"r"(su32(&empty[s])), "r"(par) : "memory");
            }
            if (lane == 0)
                asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&full[s])), "r"(tx) : "memory");
            __syncwarp();
            if (lane < ops) {
                uint32_t h = hash32(seed + i * 131 + lane);
                uint32_t dst = su32(ring + s * stage_bytes + lane * ((op_bytes + 127) / 128 * 128));
                if (mode == 0) {
                    int r0 = hash32(h) % K, r1 = hash32(h + 1) % K, r2 = hash32(h + 2) % K, r3 = hash32(h + 3) % K;
                    asm volatile(
                        "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
                        ::"r"(dst), "l"(&map), "r"(0), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(su32(&full[s])) : "memory");
                } else {
                    const uint8_t* src = B + (int64_t)(hash32(h) % K) * row_bytes;
                    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                                 ::"r"(dst), "l"(src), "r"(row_bytes), "r"(su32(&full[s])) : "memory");
                }
            }
        }
    } else if (warp == 1) {
        int acc = 0;
        for (int i = 0; i < iters; ++i) {
            const int s = i % R;
            uint32_t par = (i / R) & 1;
            asm volatile("{\n.reg .pred p;\nW2: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W2;\n}\n" ::"r"(su32(&full[s])), "r"(par) : "memory");
            acc += ring[s * stage_bytes + lane * 4];
            __syncwarp();
            if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&empty[s])) : "memory");
        }
        if (acc == 12345) sink[0] = acc;
    }
}

typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                             const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                             CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

// returns ms; *bytes = payload bytes moved
extern "C" float gather_bw2(const void* B, int K, int row_bytes, int mode, int ops, int R, int ctas, int iters, int* sink,
                            double* bytes) {
    EncodeFn enc = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&enc, cudaEnableDefault, &q);
    CUtensorMap map;
    cuuint64_t dims[2] = {(cuuint64_t)(row_bytes / 8), (cuuint64_t)K};
    cuuint64_t strides[1] = {(cuuint64_t)row_bytes};
    cuuint32_t box[2] = {(cuuint32_t)((row_bytes + 16) / 8), 1};
    cuuint32_t estr[2] = {1, 1};
    if (enc(&map, CU_TENSOR_MAP_DATA_TYPE_INT64, 2, const_cast<void*>(B), dims, strides, box, estr,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
        return -1.f;
    const int rows_per_op = mode == 0 ? 4 : 1;
    const int op_bytes = rows_per_op * (row_bytes + 16);
    const size_t smem = (size_t)R * ops * ((op_bytes + 127) / 128 * 128) + 256;
    if (cudaFuncSetAttribute(k_gather, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess) return -2.f;
    k_gather<<<ctas, 64, smem>>>(map, (const uint8_t*)B, K, row_bytes, mode, ops, R, 50, sink);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    cudaEventRecord(a);
    k_gather<<<ctas, 64, smem>>>(map, (const uint8_t*)B, K, row_bytes, mode, ops, R, iters, sink);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    if (cudaGetLastError() != cudaSuccess) return -3.f;
    *bytes = (double)ctas * iters * ops * rows_per_op * row_bytes;
    return ms;
}
