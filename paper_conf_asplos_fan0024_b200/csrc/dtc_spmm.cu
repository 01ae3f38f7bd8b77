// dtc_spmm.cu -- S1-S5: the DTC-SpMM runtime kernel re-designed for sm_100a.
//
// Paper design (Alg. 2): one thread block per 16-row window
// iterating its TC blocks: FetchSpAsync (A tile -> smem, cp.async double
// buffered), VFetchDense (B rows -> registers with LDG.128, no smem,
// P:297-301), mma m16n8k4 TF32 and a register remapping that lets each
// thread load 4 consecutive B columns and un-permutes C at the store;
// strict balance hands fixed TC-block counts to thread blocks with atomics.
//
// This kernel keeps what still holds on B200 and changes the rest:
//  * Work: a CTA takes one F4 work unit (a window-ordered run of ~U TC blocks,
//    whole windows, or one piece of a long window) x one slice of N columns.
//    The hardware CTA scheduler dispatches units in index = window order as slots
//    free up, which gives both load balance and the L2 locality of a
//    contiguous wave.  Split windows finish with a DETERMINISTIC fixup:
//    pieces write partials to a workspace, the last arriver sums them in piece
//    order (no float atomics, so C is bit-identical run to run).
//  * S1 FetchSparse: the warps of the CTA cooperatively scatter the next chunk of
//    S TC blocks into smem already in mma-fragment order (one LDS.128 / LDS.64
//    per lane per block, conflict-free), rounding A to TF32 (cvt.rna) once.
//  * S2 gather B: each thread issues one 16-byte load from each of its two B rows
//    per TC block straight into registers (shared-memory bypassing) with a
//    P-deep register prefetch ring (latency hiding instead of the paper's
//    2-buffer A pipeline).  -1 padded columns load zeros (C6).
//  * S3 mma.sync m16n8k8 (TF32) / m16n8k8 (FP16) per TC block: one instruction
//    per 8 output columns consumes a whole 16x8 TC block (k = 8).
//  * S4 epilogue: the paper's remapping generalised to k8: a thread ends up
//    owning 2*NJ consecutive columns of rows g and g+8 -> float4 stores.
//  * Accumulators stay in registers (a window's C tile is 16 x COLW per warp).
#include <cuda_fp16.h>

#include <algorithm>
#include <climits>

#include "dtc_internal.h"

namespace dtc {

constexpr int kChunk = 32;   // TC blocks staged per smem chunk (S)
constexpr int kPrefetch = 4; // B prefetch depth (TC blocks in flight per warp)

template <int DT>
struct Traits;
template <>
struct Traits<DTC_TF32> {
    static constexpr int NJ = 4;          // n8 mmas per TC block per warp
    static constexpr int COLW = 32;       // columns per warp
    static constexpr int VW = 4;          // elements per 16-byte vector
    static constexpr int FRAG_WORDS = 4;  // A fragment 32-bit words per lane
    using elt = float;
};
template <>
struct Traits<DTC_FP16> {
    static constexpr int NJ = 8;
    static constexpr int COLW = 64;
    static constexpr int VW = 8;
    static constexpr int FRAG_WORDS = 2;
    using elt = __half;
};

__device__ __forceinline__ uint32_t to_tf32(float x) {
    uint32_t r;
    asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(x));
    return r;
}

__device__ __forceinline__ void mma_tf32(float (&d)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1) {
    asm volatile(
        "mma.sync.aligned.m16n8k8.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
        "{%0,%1,%2,%3};\n"
        : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
        : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}

__device__ __forceinline__ void mma_f16(float (&d)[4], const uint32_t (&a)[2], uint32_t b) {
    asm volatile(
        "mma.sync.aligned.m16n8k8.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5}, {%6}, {%0,%1,%2,%3};\n"
        : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
        : "r"(a[0]), "r"(a[1]), "r"(b));
}

// Fragment slot of local id (row r = id>>3, col c = id&7) inside a lane-major tile:
//  TF32 m16n8k8 A: a0=(g,t) a1=(g+8,t) a2=(g,t+4) a3=(g+8,t+4), lane = 4g+t
//  FP16 m16n8k8 A: reg0=(g,2t),(g,2t+1)  reg1=(g+8,2t),(g+8,2t+1), lane = 4g+t
template <int DT>
__device__ __forceinline__ int frag_slot(int id) {
    const int r = id >> 3, c = id & 7;
    if (DT == DTC_TF32) {
        const int lane = ((r & 7) << 2) | (c & 3);
        return lane * 4 + ((r >> 3) | ((c >> 2) << 1));
    } else {
        const int lane = ((r & 7) << 2) | (c >> 1);
        return lane * 4 + (((r >> 3) << 1) | (c & 1));  // in halves
    }
}

struct alignas(16) V16 {
    uint32_t w[4];
};

template <int DT, bool VEC>
__device__ __forceinline__ V16 load_b(const void* __restrict__ B, int64_t ldb, int row, int64_t col, int64_t N) {
    V16 v;
    v.w[0] = v.w[1] = v.w[2] = v.w[3] = 0u;
    if (row < 0) return v;
    using E = typename Traits<DT>::elt;
    const E* p = reinterpret_cast<const E*>(B) + (int64_t)row * ldb + col;
    if (VEC) {
        if (col < N) {
            uint4 x = __ldg(reinterpret_cast<const uint4*>(p));
            v.w[0] = x.x; v.w[1] = x.y; v.w[2] = x.z; v.w[3] = x.w;
        }
    } else {
        if (DT == DTC_TF32) {
            const float* q = reinterpret_cast<const float*>(p);
#pragma unroll
            for (int e = 0; e < 4; ++e) v.w[e] = (col + e < N) ? __float_as_uint(__ldg(q + e)) : 0u;
        } else {
            const unsigned short* q = reinterpret_cast<const unsigned short*>(p);
#pragma unroll
            for (int e = 0; e < 8; ++e) {
                uint32_t h = (col + e < N) ? (uint32_t)__ldg(q + e) : 0u;
                v.w[e >> 1] |= h << (16 * (e & 1));
            }
        }
    }
    return v;
}

template <int DT, int WARPS, bool VEC>
__global__ void __launch_bounds__(WARPS * 32)
k_spmm(const Unit* __restrict__ units, const int32_t* __restrict__ rwo, const int32_t* __restrict__ tco,
       const uint8_t* __restrict__ lid, const int32_t* __restrict__ atob, const void* __restrict__ avals,
       const void* __restrict__ B, int64_t ldb, float* __restrict__ C, int64_t ldc, int64_t M, int64_t N,
       float* __restrict__ ws, int32_t* __restrict__ counters, int64_t npad) {
    using Tr = Traits<DT>;
    constexpr int NJ = Tr::NJ, COLW = Tr::COLW, VW = Tr::VW, FW = Tr::FRAG_WORDS;
    constexpr int P = kPrefetch;
    extern __shared__ __align__(16) uint32_t smem[];
    uint32_t* s_frag = smem;                                       // [kChunk][32*FW]
    int32_t* s_ids = reinterpret_cast<int32_t*>(smem + kChunk * 32 * FW);  // [kChunk][8]
    __shared__ int s_last;

    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int g = lane >> 2, t = lane & 3;
    const Unit u = units[blockIdx.x];
    const int64_t n0 = ((int64_t)blockIdx.y * WARPS + warp) * COLW;  // this warp's first column
    const bool active = n0 < N;
    const int64_t bcol = n0 + (int64_t)VW * g;                        // column of this thread's B vector
    const int64_t ccol = n0 + 2 * NJ * t;                             // first C column owned
    const int rsel0 = (DT == DTC_TF32) ? t : 2 * t;                   // B rows (k) this thread loads
    const int rsel1 = (DT == DTC_TF32) ? t + 4 : 2 * t + 1;
    const bool split = u.split_id >= 0;

    float acc[NJ][4];
#pragma unroll
    for (int j = 0; j < NJ; ++j) acc[j][0] = acc[j][1] = acc[j][2] = acc[j][3] = 0.f;

    auto store_window = [&](int64_t w, bool zero) {
        if (!active) return;
#pragma unroll
        for (int half = 0; half < 2; ++half) {
            const int64_t row = w * kWindow + g + 8 * half;
            if (row >= M) continue;
            float* crow = C + row * ldc;
#pragma unroll
            for (int hi = 0; hi < 2; ++hi) {        // columns ccol + hi*NJ + [0, NJ)
#pragma unroll
                for (int q = 0; q < NJ / 4; ++q) {
                    const int64_t c = ccol + hi * NJ + 4 * q;
                    float4 v;
                    v.x = zero ? 0.f : acc[4 * q + 0][2 * half + hi];
                    v.y = zero ? 0.f : acc[4 * q + 1][2 * half + hi];
                    v.z = zero ? 0.f : acc[4 * q + 2][2 * half + hi];
                    v.w = zero ? 0.f : acc[4 * q + 3][2 * half + hi];
                    if (VEC) {
                        if (c < N) *reinterpret_cast<float4*>(crow + c) = v;
                    } else {
                        if (c + 0 < N) crow[c + 0] = v.x;
                        if (c + 1 < N) crow[c + 1] = v.y;
                        if (c + 2 < N) crow[c + 2] = v.z;
                        if (c + 3 < N) crow[c + 3] = v.w;
                    }
                }
            }
        }
    };

    // window cursor over [u.wb, u.we); leading empty windows get zero rows
    int64_t cur = u.wb;
    int64_t next_end = INT_MAX;
    if (!split) {
        while (cur < u.we && rwo[cur + 1] <= u.bb) { store_window(cur, true); ++cur; }
        next_end = cur < u.we ? rwo[cur + 1] : INT_MAX;
    }

    for (int64_t cb = u.bb; cb < u.be; cb += kChunk) {
        const int nblk = (u.be - cb) < kChunk ? (int)(u.be - cb) : kChunk;
        // ---- S1: stage A tiles of this chunk in fragment order + the B row ids
        for (int j = warp; j < nblk; j += WARPS) {
            const int64_t b = cb + j;
            const int lo = tco[b], hi = tco[b + 1];
            uint32_t* fr = s_frag + j * 32 * FW;
            if (FW == 4) reinterpret_cast<uint4*>(fr)[lane] = make_uint4(0u, 0u, 0u, 0u);
            else reinterpret_cast<uint2*>(fr)[lane] = make_uint2(0u, 0u);
            if (lane < 8) s_ids[j * 8 + lane] = atob[b * 8 + lane];
            __syncwarp();
            for (int e = lo + lane; e < hi; e += 32) {
                const int id = lid[e];
                const int slot = frag_slot<DT>(id);
                if (DT == DTC_TF32) {
                    fr[slot] = to_tf32(reinterpret_cast<const float*>(avals)[e]);
                } else {
                    reinterpret_cast<unsigned short*>(fr)[slot] = reinterpret_cast<const unsigned short*>(avals)[e];
                }
            }
        }
        __syncthreads();
        // ---- S2/S3: gather B into registers P blocks ahead, mma per TC block
        if (active) {
            V16 b0[P], b1[P];
#pragma unroll
            for (int q = 0; q < P; ++q) {
                if (q < nblk) {
                    b0[q] = load_b<DT, VEC>(B, ldb, s_ids[q * 8 + rsel0], bcol, N);
                    b1[q] = load_b<DT, VEC>(B, ldb, s_ids[q * 8 + rsel1], bcol, N);
                }
            }
            for (int j0 = 0; j0 < nblk; j0 += P) {
#pragma unroll
                for (int q = 0; q < P; ++q) {
                    const int j = j0 + q;
                    if (j < nblk) {
                        const uint32_t* fr = s_frag + j * 32 * FW;
                        if (DT == DTC_TF32) {
                            const uint4 av = reinterpret_cast<const uint4*>(fr)[lane];
                            const uint32_t a[4] = {av.x, av.y, av.z, av.w};
#pragma unroll
                            for (int jj = 0; jj < NJ; ++jj)
                                mma_tf32(acc[jj], a, to_tf32(__uint_as_float(b0[q].w[jj])),
                                         to_tf32(__uint_as_float(b1[q].w[jj])));
                        } else {
                            const uint2 av = reinterpret_cast<const uint2*>(fr)[lane];
                            const uint32_t a[2] = {av.x, av.y};
#pragma unroll
                            for (int jj = 0; jj < NJ; ++jj) {
                                const uint32_t bb = __byte_perm(b0[q].w[jj >> 1], b1[q].w[jj >> 1],
                                                                (jj & 1) ? 0x7632 : 0x5410);
                                mma_f16(acc[jj], a, bb);
                            }
                        }
                        if (j + P < nblk) {
                            b0[q] = load_b<DT, VEC>(B, ldb, s_ids[(j + P) * 8 + rsel0], bcol, N);
                            b1[q] = load_b<DT, VEC>(B, ldb, s_ids[(j + P) * 8 + rsel1], bcol, N);
                        }
                        // ---- S4: window boundary -> store and reset
                        const int64_t b = cb + j;
                        if (b + 1 == next_end) {
                            store_window(cur, false);
#pragma unroll
                            for (int jj = 0; jj < NJ; ++jj) acc[jj][0] = acc[jj][1] = acc[jj][2] = acc[jj][3] = 0.f;
                            ++cur;
                            while (cur < u.we && rwo[cur + 1] == rwo[cur]) { store_window(cur, true); ++cur; }
                            next_end = cur < u.we ? rwo[cur + 1] : INT_MAX;
                        }
                    }
                }
            }
        }  // inactive warps (columns >= N) only help stage A; they store nothing
        __syncthreads();
    }

    if (!split) {
        while (cur < u.we) { store_window(cur, true); ++cur; }
        return;
    }

    // ---- S5: split-window fixup (deterministic: partials summed in piece order)
    const int64_t slot = (int64_t)u.slot_base + u.piece;
    if (active) {
#pragma unroll
        for (int half = 0; half < 2; ++half) {
            float* prow = ws + (slot * kWindow + g + 8 * half) * npad;
#pragma unroll
            for (int hi = 0; hi < 2; ++hi)
#pragma unroll
                for (int q = 0; q < NJ / 4; ++q) {
                    const int64_t c = ccol + hi * NJ + 4 * q;
                    float4 v = make_float4(acc[4 * q + 0][2 * half + hi], acc[4 * q + 1][2 * half + hi],
                                           acc[4 * q + 2][2 * half + hi], acc[4 * q + 3][2 * half + hi]);
                    __stcg(reinterpret_cast<float4*>(prow + c), v);
                }
        }
    }
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) {
        int32_t* ctr = counters + (int64_t)u.split_id * gridDim.y + blockIdx.y;
        const int prev = atomicAdd(ctr, 1);
        s_last = (prev == u.npieces - 1);
        if (s_last) *ctr = 0;  // self-reset for the next launch (stream-ordered)
    }
    __syncthreads();
    if (!s_last) return;
    __threadfence();
#pragma unroll
    for (int j = 0; j < NJ; ++j) acc[j][0] = acc[j][1] = acc[j][2] = acc[j][3] = 0.f;
    if (!active) return;
    for (int pc = 0; pc < u.npieces; ++pc) {
        const int64_t sl = (int64_t)u.slot_base + pc;
#pragma unroll
        for (int half = 0; half < 2; ++half) {
            const float* prow = ws + (sl * kWindow + g + 8 * half) * npad;
#pragma unroll
            for (int hi = 0; hi < 2; ++hi)
#pragma unroll
                for (int q = 0; q < NJ / 4; ++q) {
                    const int64_t c = ccol + hi * NJ + 4 * q;
                    const float4 v = __ldcg(reinterpret_cast<const float4*>(prow + c));
                    acc[4 * q + 0][2 * half + hi] += v.x;
                    acc[4 * q + 1][2 * half + hi] += v.y;
                    acc[4 * q + 2][2 * half + hi] += v.z;
                    acc[4 * q + 3][2 * half + hi] += v.w;
                }
        }
    }
    store_window(u.wb, false);
}

template <int DT, int WARPS, bool VEC>
static cudaError_t launch_one(dtc_format* h, const void* B, int64_t ldb, float* C, int64_t ldc, int64_t N,
                              int gy, int64_t npad, cudaStream_t s) {
    using Tr = Traits<DT>;
    const size_t smem = (size_t)kChunk * 32 * Tr::FRAG_WORDS * 4 + (size_t)kChunk * 8 * 4;
    dim3 grid((unsigned)h->num_units, (unsigned)gy);
    k_spmm<DT, WARPS, VEC><<<grid, WARPS * 32, smem, s>>>(h->units, h->rwo, h->tco, h->lid, h->atob, h->vals, B,
                                                          ldb, C, ldc, h->M, N, h->ws, h->counters, npad);
    return cudaGetLastError();
}

template <int DT, bool VEC>
static cudaError_t dispatch_warps(int warps, dtc_format* h, const void* B, int64_t ldb, float* C, int64_t ldc,
                                  int64_t N, int gy, int64_t npad, cudaStream_t s) {
    switch (warps) {
        case 1: return launch_one<DT, 1, VEC>(h, B, ldb, C, ldc, N, gy, npad, s);
        case 2: return launch_one<DT, 2, VEC>(h, B, ldb, C, ldc, N, gy, npad, s);
        case 4: return launch_one<DT, 4, VEC>(h, B, ldb, C, ldc, N, gy, npad, s);
        default: return launch_one<DT, 8, VEC>(h, B, ldb, C, ldc, N, gy, npad, s);
    }
}

int spmm_launch(dtc_format* h, const void* B, int64_t N, int64_t ldb, float* C, int64_t ldc, cudaStream_t s) {
    if (!h) { set_error("null handle"); return DTC_ERR_INVALID; }
    if (N < 1 || ldb < N || ldc < N) { set_error("bad N/ldb/ldc (%lld/%lld/%lld)", (long long)N, (long long)ldb, (long long)ldc); return DTC_ERR_INVALID; }
    if (h->M == 0) return DTC_OK;
    if (!C || (!B && h->T > 0)) { set_error("null B or C"); return DTC_ERR_INVALID; }
    if (h->num_units == 0) return DTC_OK;
    const int elt = elt_size(h->dtype);
    const int VW = 16 / elt;
    const bool vec = ((uintptr_t)B % 16 == 0) && ((uintptr_t)C % 16 == 0) && (ldb % VW == 0) && (N % VW == 0) &&
                     (ldc % 4 == 0);
    const int colw = h->dtype == DTC_FP16 ? Traits<DTC_FP16>::COLW : Traits<DTC_TF32>::COLW;
    const int64_t need = (N + colw - 1) / colw;
    const int warps = need >= 8 ? 8 : need >= 4 ? 4 : need >= 2 ? (need > 2 ? 4 : 2) : 1;
    const int64_t gy64 = (N + (int64_t)warps * colw - 1) / ((int64_t)warps * colw);
    if (gy64 > 65535) { set_error("N too large"); return DTC_ERR_UNSUPPORTED; }
    const int gy = (int)gy64;
    const int64_t npad = gy64 * warps * colw;
    // split-window state
    if (h->num_split > 0) {
        const int64_t ncnt = h->num_split * gy;
        if (ncnt > h->counters_len) {
            dfree(h->counters, s);
            h->counters_len = 0;
            int rc = dalloc(&h->counters, ncnt, s);
            if (rc) return rc;
            DTC_CUDA(cudaMemsetAsync(h->counters, 0, ncnt * sizeof(int32_t), s));
            h->counters_len = ncnt;
        }
        const size_t wsb = (size_t)h->num_slots * kWindow * npad * sizeof(float);
        if (wsb > h->ws_bytes) {
            dfree(h->ws, s);
            h->ws_bytes = 0;
            int rc = dalloc(&h->ws, wsb / sizeof(float), s);
            if (rc) return rc;
            h->ws_bytes = wsb;
        }
    }
    cudaError_t e;
    if (h->dtype == DTC_FP16)
        e = vec ? dispatch_warps<DTC_FP16, true>(warps, h, B, ldb, C, ldc, N, gy, npad, s)
                : dispatch_warps<DTC_FP16, false>(warps, h, B, ldb, C, ldc, N, gy, npad, s);
    else
        e = vec ? dispatch_warps<DTC_TF32, true>(warps, h, B, ldb, C, ldc, N, gy, npad, s)
                : dispatch_warps<DTC_TF32, false>(warps, h, B, ldb, C, ldc, N, gy, npad, s);
    if (e != cudaSuccess) return cuda_fail(e, "k_spmm launch", __FILE__, __LINE__);
    return DTC_OK;
}

}  // namespace dtc

using namespace dtc;

extern "C" int dtc_spmm(dtc_handle_t h, const void* B, int64_t N, int64_t ldb, float* C, int64_t ldc, void* stream) {
    return spmm_launch(h, B, N, ldb, C, ldc, (cudaStream_t)stream);
}

extern "C" int dtc_spmm_launches_per_call(void) { return 1; }

extern "C" int dtc_spmm_host(dtc_handle_t h, const void* B_host, int64_t N, int64_t ldb, float* C_host,
                             int64_t ldc, void* stream) {
    if (!h || !C_host || (!B_host && h->K > 0)) { set_error("null argument"); return DTC_ERR_INVALID; }
    if (N < 1 || ldb < N || ldc < N) { set_error("bad N/ldb/ldc"); return DTC_ERR_INVALID; }
    cudaStream_t s = (cudaStream_t)stream;
    const int elt = elt_size(h->dtype);
    const size_t bbytes = (size_t)std::max<int64_t>(h->K, 1) * N * elt;
    const size_t cbytes = (size_t)std::max<int64_t>(h->M, 1) * N * sizeof(float);
    if (bbytes > h->stage_B_bytes) {
        dfree(h->stage_B, s);
        h->stage_B_bytes = 0;
        DTC_CUDA(cudaMallocAsync(&h->stage_B, bbytes, s));
        h->stage_B_bytes = bbytes;
    }
    if (cbytes > h->stage_C_bytes) {
        dfree(h->stage_C, s);
        h->stage_C_bytes = 0;
        DTC_CUDA(cudaMallocAsync((void**)&h->stage_C, cbytes, s));
        h->stage_C_bytes = cbytes;
    }
    if (h->K > 0)
        DTC_CUDA(cudaMemcpy2DAsync(h->stage_B, N * elt, B_host, ldb * elt, N * elt, h->K, cudaMemcpyHostToDevice, s));
    int rc = spmm_launch(h, h->stage_B, N, N, h->stage_C, N, s);
    if (rc) return rc;
    if (h->M > 0)
        DTC_CUDA(cudaMemcpy2DAsync(C_host, ldc * sizeof(float), h->stage_C, N * sizeof(float), N * sizeof(float), h->M,
                                   cudaMemcpyDeviceToHost, s));
    DTC_CUDA(cudaStreamSynchronize(s));
    return DTC_OK;
}
