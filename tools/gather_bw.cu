// gather_bw.cu -- microbenchmark (not product code): throughput of row gathers
// on sm_100a, to choose the B-gather mechanism of the SpMM kernel.
//   mode 0: TMA tile::gather4, box = {box_cols, 1}, 1 thread issues ops_per_stage ops per stage
//   mode 1: warp LDG.128, fragment order (4 rows per 8 lanes)   -- the v1 kernel's pattern
//   mode 2: warp LDG.128, coalesced (8 lanes per row)
//   mode 3: cp.async 16B (LDGSTS), coalesced, per-warp ring
// Rows are pseudo-random over a K x ldb fp32 matrix.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>

__device__ __forceinline__ uint32_t hash32(uint32_t x) {
    x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16;
    return x;
}
__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void k_tma(const __grid_constant__ CUtensorMap map, int K, int ncolbox, int box_bytes, int ops_per_stage,
                      int R, int iters, int* sink) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ __align__(8) uint64_t full[32], empty[32];
    uint8_t* ring = (uint8_t*)(((uintptr_t)sm + 1023) & ~(uintptr_t)1023);
    const int stage_bytes = ops_per_stage * 4 * box_bytes;
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
    if (warp == 0) {  // producer: lanes < ops_per_stage each issue one gather4
        for (int i = 0; i < iters; ++i) {
            const int s = i % R;
            if (i >= R) {
                uint32_t par = ((i / R) - 1) & 1;
                asm volatile("{\n.reg .pred p;\nW1: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W1;\n}\n" ::"r"(su32(&empty[s])), "r"(par) : "memory");
            }
            if (lane == 0)
                asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&full[s])), "r"(stage_bytes) : "memory");
            __syncwarp();
            if (lane < ops_per_stage) {
                uint32_t h = hash32(seed + i * 131 + lane);
                int r0 = hash32(h) % K, r1 = hash32(h + 1) % K, r2 = hash32(h + 2) % K, r3 = hash32(h + 3) % K;
                int col = (lane % ncolbox) * (box_bytes / 4);
                uint32_t dst = su32(ring + s * stage_bytes + lane * 4 * box_bytes);
                asm volatile(
                    "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
                    ::"r"(dst), "l"(&map), "r"(col), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(su32(&full[s])) : "memory");
            }
        }
    } else if (warp == 1) {  // consumer
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

// LDG: each warp loads 8 rows x 128 B per "block" with 2 LDG.128 per thread, depth P in registers.
template <int MODE, int P>
__global__ void k_ldg(const float* __restrict__ B, int K, int ldb, int iters, int* sink) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int g = lane >> 2, t = lane & 3;
    uint32_t seed = (blockIdx.x * 64 + warp) * 7919u;
    float4 v0[P], v1[P];
    float acc = 0.f;
    auto rows = [&](int i, int& ra, int& rb) {
        uint32_t h = hash32(seed + i * 131);
        if (MODE == 1) { ra = hash32(h + t) % K; rb = hash32(h + t + 4) % K; }
        else { ra = hash32(h + (lane >> 3)) % K; rb = hash32(h + 4 + (lane >> 3)) % K; }
    };
    auto colof = [&]() { return MODE == 1 ? 4 * g : 4 * (lane & 7); };
#pragma unroll
    for (int q = 0; q < P; ++q) {
        int ra, rb; rows(q, ra, rb);
        v0[q] = __ldg(reinterpret_cast<const float4*>(B + (int64_t)ra * ldb + colof()));
        v1[q] = __ldg(reinterpret_cast<const float4*>(B + (int64_t)rb * ldb + colof()));
    }
    for (int i0 = 0; i0 < iters; i0 += P) {
#pragma unroll
        for (int q = 0; q < P; ++q) {
            acc += v0[q].x + v1[q].y;
            int ra, rb; rows(i0 + q + P, ra, rb);
            v0[q] = __ldg(reinterpret_cast<const float4*>(B + (int64_t)ra * ldb + colof()));
            v1[q] = __ldg(reinterpret_cast<const float4*>(B + (int64_t)rb * ldb + colof()));
        }
    }
    if (acc == 1234.5f) sink[0] = 1;
}

// cp.async 16B per thread, coalesced rows, per-warp ring of D stages (1 KB each)
template <int D>
__global__ void k_cpasync(const float* __restrict__ B, int K, int ldb, int iters, int* sink) {
    extern __shared__ __align__(16) uint8_t sm[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    uint8_t* ring = sm + warp * D * 1024;
    uint32_t seed = (blockIdx.x * 64 + warp) * 7919u;
    float acc = 0.f;
    auto issue = [&](int i) {
        uint32_t h = hash32(seed + i * 131);
        int ra = hash32(h + (lane >> 3)) % K, rb = hash32(h + 4 + (lane >> 3)) % K;
        const float* sa = B + (int64_t)ra * ldb + 4 * (lane & 7);
        const float* sb = B + (int64_t)rb * ldb + 4 * (lane & 7);
        uint32_t d = su32(ring + (i % D) * 1024 + lane * 16);
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d), "l"(sa));
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d + 512), "l"(sb));
        asm volatile("cp.async.commit_group;");
    };
    for (int q = 0; q < D - 1; ++q) issue(q);
    for (int i = 0; i < iters; ++i) {
        issue(i + D - 1);
        asm volatile("cp.async.wait_group %0;" ::"n"(D - 1));
        __syncwarp();
        acc += *reinterpret_cast<const float*>(ring + (i % D) * 1024 + lane * 16);
        __syncwarp();
    }
    asm volatile("cp.async.wait_all;");
    if (acc == 1234.5f) sink[0] = 1;
}

typedef CUresult (*EncodeTiled)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

extern "C" float gather_bw(int mode, const float* B, int K, int ldb, int box_cols, int swizzle, int ops_per_stage,
                           int R, int ctas, int threads, int iters, int* sink, double* bytes_out) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    double bytes = 0;
    if (mode == 0) {
        EncodeTiled enc;
        cudaDriverEntryPointQueryResult q;
        cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&enc, cudaEnableDefault, &q);
        CUtensorMap map;
        cuuint64_t dims[2] = {(cuuint64_t)ldb, (cuuint64_t)K};
        cuuint64_t str[1] = {(cuuint64_t)ldb * 4};
        cuuint32_t box[2] = {(cuuint32_t)box_cols, 1}, es[2] = {1, 1};
        enc(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, (void*)B, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
            swizzle ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        int box_bytes = box_cols * 4;
        int ncolbox = ldb / box_cols;
        size_t smem = 1024 + (size_t)R * ops_per_stage * 4 * box_bytes;
        cudaFuncSetAttribute(k_tma, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        k_tma<<<ctas, 64, smem>>>(map, K, ncolbox, box_bytes, ops_per_stage, R, 4, sink);
        cudaEventRecord(a);
        k_tma<<<ctas, 64, smem>>>(map, K, ncolbox, box_bytes, ops_per_stage, R, iters, sink);
        cudaEventRecord(b);
        bytes = (double)ctas * iters * ops_per_stage * 4 * box_bytes;
    } else if (mode == 1 || mode == 2) {
        auto kern = mode == 1 ? k_ldg<1, 4> : k_ldg<2, 4>;
        kern<<<ctas, threads>>>(B, K, ldb, 8, sink);
        cudaEventRecord(a);
        kern<<<ctas, threads>>>(B, K, ldb, iters, sink);
        cudaEventRecord(b);
        bytes = (double)ctas * (threads / 32) * (iters + 4) * 1024;
    } else {
        size_t smem = (size_t)(threads / 32) * 8 * 1024;
        cudaFuncSetAttribute(k_cpasync<8>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        k_cpasync<8><<<ctas, threads, smem>>>(B, K, ldb, 8, sink);
        cudaEventRecord(a);
        k_cpasync<8><<<ctas, threads, smem>>>(B, K, ldb, iters, sink);
        cudaEventRecord(b);
        bytes = (double)ctas * (threads / 32) * (iters + 7) * 1024;
    }
    cudaEventSynchronize(b);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); return -1; }
    *bytes_out = bytes;
    return ms;
}
