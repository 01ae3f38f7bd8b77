// tma_probe.cu -- hardware probe (not product code): behaviour of
// cp.async.bulk.tensor.2d.tile::gather4 on sm_100a -- tensor-map box shape,
// 128B-swizzle layout and zero fill for out-of-bounds row coordinates.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>

typedef CUresult (*EncodeTiled)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

__global__ void probe_kernel(const __grid_constant__ CUtensorMap map, int col0, int r0, int r1, int r2, int r3,
                             int bytes, uint32_t* out) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ __align__(8) uint64_t bar;
    uint32_t b = (uint32_t)__cvta_generic_to_shared(&bar);
    uint32_t d = (uint32_t)__cvta_generic_to_shared(sm);
    for (int i = threadIdx.x; i < 4096 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(sm)[i] = 0xDEADBEEFu;
    __syncthreads();
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(b));
        asm volatile("fence.proxy.async.shared::cta;");
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(bytes));
        asm volatile(
            "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, "
            "%4, %5, %6}], [%7];" ::"r"(d),
            "l"(&map), "r"(col0), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(b)
            : "memory");
        asm volatile(
            "{\n.reg .pred p;\nW: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n@!p bra W;\n}\n" ::"r"(b)
            : "memory");
    }
    __syncthreads();
    for (int i = threadIdx.x; i < 4096 / 4; i += blockDim.x) out[i] = reinterpret_cast<uint32_t*>(sm)[i];
}

extern "C" int tma_probe(const void* B, int64_t K, int64_t N, int elt, int box_cols, int box_rows, int swizzle,
                         int col0, int r0, int r1, int r2, int r3, uint32_t* out_dev, char* msg) {
    EncodeTiled enc = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&enc, cudaEnableDefault, &q) != cudaSuccess || !enc) {
        sprintf(msg, "no cuTensorMapEncodeTiled");
        return -1;
    }
    CUtensorMap map;
    cuuint64_t dims[2] = {(cuuint64_t)N, (cuuint64_t)K};
    cuuint64_t strides[1] = {(cuuint64_t)(N * elt)};
    cuuint32_t box[2] = {(cuuint32_t)box_cols, (cuuint32_t)box_rows};
    cuuint32_t estr[2] = {1, 1};
    CUtensorMapSwizzle sw = swizzle == 128 ? CU_TENSOR_MAP_SWIZZLE_128B
                            : swizzle == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                            : swizzle == 32 ? CU_TENSOR_MAP_SWIZZLE_32B
                                            : CU_TENSOR_MAP_SWIZZLE_NONE;
    CUresult r = enc(&map, elt == 4 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, (void*)B,
                     dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) {
        sprintf(msg, "encode failed %d", (int)r);
        return -2;
    }
    int bytes = 4 * box_cols * elt;
    probe_kernel<<<1, 128, 8192>>>(map, col0, r0, r1, r2, r3, bytes, out_dev);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) {
        sprintf(msg, "kernel: %s", cudaGetErrorString(e));
        return -3;
    }
    sprintf(msg, "ok");
    return 0;
}
