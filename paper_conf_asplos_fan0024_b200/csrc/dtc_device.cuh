// dtc_device.cuh -- small device helpers shared by the builder kernels.
#pragma once
#include <cstdint>

namespace dtc {

// Block-wide exclusive scan for blockDim.x == NT (multiple of 32, <= 1024).
// Returns the exclusive prefix of v; *total gets the block sum.  Contains
// __syncthreads(): every thread of the block must call it.
template <int NT, class T>
__device__ __forceinline__ T block_exscan(T v, T* total) {
    __shared__ T warp_sums[NT / 32];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    T x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        T y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) warp_sums[warp] = x;
    __syncthreads();
    if (warp == 0) {
        T w = lane < NT / 32 ? warp_sums[lane] : T(0);
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            T y = __shfl_up_sync(0xffffffffu, w, o);
            if (lane >= o) w += y;
        }
        if (lane < NT / 32) warp_sums[lane] = w;
    }
    __syncthreads();
    T base = warp > 0 ? warp_sums[warp - 1] : T(0);
    *total = warp_sums[NT / 32 - 1];
    __syncthreads();
    return base + x - v;
}

template <int NT>
__device__ __forceinline__ int block_min(int v) {
    __shared__ int red[NT / 32];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = min(v, __shfl_xor_sync(0xffffffffu, v, o));
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = v;
    __syncthreads();
    int r = red[0];
#pragma unroll
    for (int i = 1; i < NT / 32; ++i) r = min(r, red[i]);
    __syncthreads();
    return r;
}

template <int NT>
__device__ __forceinline__ int block_max(int v) {
    __shared__ int red[NT / 32];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = max(v, __shfl_xor_sync(0xffffffffu, v, o));
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = v;
    __syncthreads();
    int r = red[0];
#pragma unroll
    for (int i = 1; i < NT / 32; ++i) r = max(r, red[i]);
    __syncthreads();
    return r;
}

}  // namespace dtc
