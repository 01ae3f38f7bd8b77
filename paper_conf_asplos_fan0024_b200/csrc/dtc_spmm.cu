// dtc_spmm.cu -- S1-S5: the DTC-SpMM runtime kernel re-designed for sm_100a.
//
// Paper design (Alg. 2): one thread block per 16-row window
// iterating its TC blocks: FetchSpAsync (A tile -> smem, cp.async double
// buffered), VFetchDense (B rows -> registers with LDG.128, bypassing
// smem), mma m16n8k4 TF32, a register remapping that lets each
// thread load 4 consecutive B columns and un-permutes C at the store,
// and strict balance of TC blocks over thread blocks with atomics.
//
// What changes on B200 (measured, profiles/r01_design_evidence.md).
// Three kernel variants compute S1-S5 with the same arithmetic (dtc_set_spmm_path):
//  * k_spmm_ldg (path 1): the CTA stages chunks of 16/32 TC blocks of A into shared
//    memory already in mma-fragment order and TF32-rounded (FetchSparse + the paper's
//    sparse double buffering, two chunks deep); every warp gathers its B rows
//    straight into registers one block ahead (the shared-memory bypass + register
//    remap of P:297-319, generalised to m16n8k8).
//  * k_spmm_dir (path 3): no shared memory and no CTA barrier: each warp builds its own
//    A fragment from TCValues through a 128-bit occupancy mask per TC block, and work
//    items (unit x column slice) run in L2-sized column passes.
//  * k_spmm_tma (path 2, ablation): B rows gathered by TMA tile::gather4 into a
//    128B-swizzled smem ring (the async global->smem gather the paper lacked);
//    measured op-rate bound at ~4 TB/s for 512-byte boxes, so it is not the default.
// Common to all: mma.sync m16n8k8 TF32/FP16 with FP32 accumulation (C22);
// balance + locality from the F4 work units (TC-block sized, window ordered, P:333,
// P:258) dispatched in order; split windows finish with a deterministic fixup
// (partials summed in piece order; no float atomics, P:333 used atomics).
#include <cuda.h>
#include <cuda_fp16.h>

#include <algorithm>
#include <climits>
#include <vector>

#include "dtc_internal.h"

namespace dtc {

constexpr int kChunk = 32;      // TC blocks per A batch (S)
// Register-gather tuning per (dtype, consumer warps): B prefetch depth P and the
// register cap that sets occupancy (measured sweep).  The A chunk
// is the largest multiple of P not above 32 TC blocks.  -DDTC_PREFETCH /
// -DDTC_LDG_MAXREGS override both for sweeps.
template <int DT, int W>
constexpr int ldg_prefetch() {
#ifdef DTC_PREFETCH
    return DTC_PREFETCH;
#else
    return 1;
#endif
}
// per-thread register cap (sets occupancy) for a CTA of W consumer warps, each owning CW column
// chunks -- from the measured sweeps (profiles/r01_design_evidence.md)
template <int DT, int W, int CW>
constexpr int ldg_maxregs() {
#ifdef DTC_LDG_MAXREGS
    return DTC_LDG_MAXREGS * CW;
#else
    return CW == 1 ? 64 : (DT == DTC_FP16 ? 112 : (W <= 2 ? 96 : 80));
#endif
}
template <int DT, int W, int CW>
constexpr int ldg_min_blocks() {
    constexpr int b = 65536 / (W * 32 * ldg_maxregs<DT, W, CW>());
    return b > 32 ? 32 : (b < 1 ? 1 : b);
}
// column chunks (of 32 fp32 / 64 fp16 columns) per consumer warp in the register-gather kernel
template <int DT>
constexpr int ldg_colchunks() {
#if defined(DTC_TF32_CW) || defined(DTC_FP16_CW)
#ifndef DTC_TF32_CW
#define DTC_TF32_CW 2
#endif
#ifndef DTC_FP16_CW
#define DTC_FP16_CW 1
#endif
    return DT == DTC_TF32 ? DTC_TF32_CW : DTC_FP16_CW;
#else
    return 2;   // a warp owns 2 x 128-byte column slices: one A-fragment read per 64 fp32 / 128 fp16 columns
#endif
}
template <int DT, int W>
constexpr int ldg_chunk_target() {
#ifdef DTC_CHUNK
    return DTC_CHUNK;
#else
    return (DT == DTC_TF32 && W <= 4) ? 16 : 32;   // smaller chunks let 8 TF32 CTAs of 4 warps fit in smem
#endif
}
template <int DT, int W>
constexpr int ldg_chunk() { return ldg_prefetch<DT, W>() * (ldg_chunk_target<DT, W>() / ldg_prefetch<DT, W>()); }

constexpr int kBRingBytes = 64 * 1024;   // TMA path: B stage ring per CTA

template <int DT>
struct Traits;
template <>
struct Traits<DTC_TF32> {
    static constexpr int NJ = 4;          // n8 mmas per TC block per warp
    static constexpr int COLW = 32;       // columns per warp (= one 128-byte row slice)
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

// ------------------------------------------------------------ mbarriers (CTA scope)
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, int count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    asm volatile(
        "{\n"
        ".reg .pred p;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        "@!p bra WAIT_%=;\n"
        "}\n" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}

// L2 eviction-priority hints (experiment DTC_L2_HINTS): B gathers evict_last, streamed data
// (C stores) evict_first, so reusable B rows survive the streaming traffic in L2.
#ifdef DTC_L2_HINTS
__device__ __forceinline__ uint64_t l2_policy_last() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t l2_policy_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint4 ldg_hint(const void* ptr, uint64_t pol) {
    uint4 r;
    asm volatile("ld.global.nc.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(ptr), "l"(pol));
    return r;
}
__device__ __forceinline__ void stg_hint(void* ptr, float4 v, uint64_t pol) {
    asm volatile("st.global.L2::cache_hint.v4.f32 [%0], {%1,%2,%3,%4}, %5;"
                 :: "l"(ptr), "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w), "l"(pol) : "memory");
}
#endif

// --------------------------------------------------- C tile store / split partials
// A consumer warp owns rows (w*16 + g, w*16 + g + 8) and, for hi in {0,1} and
// quad q < NJ/4, the 4 consecutive columns base + hi*HOFF + col_of_quad(q)
// (acc[4q..4q+3][2*half+hi]).  A warp may own CW column chunks of QPC quads each,
// CSTRIDE columns apart: col_of_quad(q) = 4*(q % QPC) + CSTRIDE*(q / QPC).
template <int QPC, int CSTRIDE>
__device__ __forceinline__ int col_of_quad(int q) { return 4 * (q % QPC) + CSTRIDE * (q / QPC); }

template <int NJ, bool VEC, int QPC = NJ / 4, int CSTRIDE = 0>
__device__ __forceinline__ void store_tile(float* __restrict__ C, int64_t ldc, int64_t M, int64_t N, int64_t w, int g,
                                           int64_t base, int hoff, const float (&acc)[NJ][4], bool zero,
                                           const int32_t* __restrict__ rowmap) {
#pragma unroll
    for (int half = 0; half < 2; ++half) {
        const int64_t row = w * kWindow + g + 8 * half;
        if (row >= M) continue;
        // row of the (possibly TCA-permuted) condensed matrix -> row of C in the caller's order
        float* crow = C + (rowmap ? (int64_t)__ldg(rowmap + row) : row) * ldc;
#pragma unroll
        for (int hi = 0; hi < 2; ++hi) {
#pragma unroll
            for (int q = 0; q < NJ / 4; ++q) {
                const int64_t c = base + hi * hoff + col_of_quad<QPC, CSTRIDE>(q);
                float4 v;
                v.x = zero ? 0.f : acc[4 * q + 0][2 * half + hi];
                v.y = zero ? 0.f : acc[4 * q + 1][2 * half + hi];
                v.z = zero ? 0.f : acc[4 * q + 2][2 * half + hi];
                v.w = zero ? 0.f : acc[4 * q + 3][2 * half + hi];
                if (VEC) {
#if defined(DTC_L2_HINTS) && (DTC_L2_HINTS & 2)
                    if (c < N) stg_hint(crow + c, v, l2_policy_first());
#elif defined(DTC_C_STORE_CS)
                    if (c < N) __stcs(reinterpret_cast<float4*>(crow + c), v);   // streaming (evict-first)
#else
                    if (c < N) *reinterpret_cast<float4*>(crow + c) = v;
#endif
                } else {
                    if (c + 0 < N) crow[c + 0] = v.x;
                    if (c + 1 < N) crow[c + 1] = v.y;
                    if (c + 2 < N) crow[c + 2] = v.z;
                    if (c + 3 < N) crow[c + 3] = v.w;
                }
            }
        }
    }
}

// Split-window fixup for one warp's tile, deterministic, two levels.  A window split into np
// pieces forms groups of G = ceil(sqrt(np)) consecutive pieces (one group when np <= 4).  Every piece
// writes its partial to its slot; the last arriving piece of a group sums the group's slots in piece
// order (into the group's first slot); the last arriving group sums the group sums in group order
// and stores C.  The chain of dependent partial loads is G + np/G instead of np (the single-level
// chain made the last arriver of a hub window the tail of the launch).  Counters live at
// ctr0[slot * cstride] (one per slot and warp column slice): group g at its first slot, the window
// at slot_base + 1 (never a group's first slot when there are >= 2 groups); all self-resetting.
__device__ __forceinline__ int fixup_group(int np) {
    if (np <= 4) return np;
    int g = 1;
    while (g * g < np) ++g;
    return g;
}

template <int NJ, int QPC, int CSTRIDE>
__device__ __forceinline__ void fixup_write(float (&acc)[NJ][4], float* __restrict__ ws, int64_t slot, int64_t npad,
                                            int g, int64_t base, int hoff) {
#pragma unroll
    for (int half = 0; half < 2; ++half) {
        float* prow = ws + (slot * kWindow + g + 8 * half) * npad;
#pragma unroll
        for (int hi = 0; hi < 2; ++hi)
#pragma unroll
            for (int q = 0; q < NJ / 4; ++q) {
                const int64_t c = base + hi * hoff + col_of_quad<QPC, CSTRIDE>(q);
                __stcg(reinterpret_cast<float4*>(prow + c),
                       make_float4(acc[4 * q + 0][2 * half + hi], acc[4 * q + 1][2 * half + hi],
                                   acc[4 * q + 2][2 * half + hi], acc[4 * q + 3][2 * half + hi]));
            }
    }
}

// acc := sum over k < cnt of slot (s0 + k * step), in k order
template <int NJ, int QPC, int CSTRIDE>
__device__ __forceinline__ void fixup_sum(float (&acc)[NJ][4], const float* __restrict__ ws, int64_t s0, int64_t step,
                                          int cnt, int64_t npad, int g, int64_t base, int hoff) {
#pragma unroll
    for (int j = 0; j < NJ; ++j) acc[j][0] = acc[j][1] = acc[j][2] = acc[j][3] = 0.f;
#pragma unroll 1
    for (int k = 0; k < cnt; ++k) {
        const int64_t sl = s0 + k * step;
#pragma unroll
        for (int half = 0; half < 2; ++half) {
            const float* prow = ws + (sl * kWindow + g + 8 * half) * npad;
#pragma unroll
            for (int hi = 0; hi < 2; ++hi)
#pragma unroll
                for (int q = 0; q < NJ / 4; ++q) {
                    const int64_t c = base + hi * hoff + col_of_quad<QPC, CSTRIDE>(q);
                    const float4 v = __ldcg(reinterpret_cast<const float4*>(prow + c));
                    acc[4 * q + 0][2 * half + hi] += v.x;
                    acc[4 * q + 1][2 * half + hi] += v.y;
                    acc[4 * q + 2][2 * half + hi] += v.z;
                    acc[4 * q + 3][2 * half + hi] += v.w;
                }
        }
    }
}

// true in every lane of the warp that arrives n-th at *ctr (the counter is reset for the next launch)
__device__ __forceinline__ bool arrive_last(int32_t* ctr, int n, int lane) {
    __threadfence();
    __syncwarp();
    int last = 0;
    if (lane == 0) {
        const int prev = atomicAdd(ctr, 1);
        last = (prev == n - 1);
        if (last) *ctr = 0;
    }
    last = __shfl_sync(0xffffffffu, last, 0);
    if (last) __threadfence();
    return last != 0;
}

template <int NJ, bool VEC, int QPC = NJ / 4, int CSTRIDE = 0>
__device__ __forceinline__ void split_fixup(const Unit& u, float (&acc)[NJ][4], float* __restrict__ ws, int64_t npad,
                                            int32_t* __restrict__ ctr0, int64_t cstride, float* __restrict__ C,
                                            int64_t ldc, int64_t M, int64_t N, int g, int lane, int64_t base, int hoff,
                                            const int32_t* __restrict__ rowmap) {
    const int np = u.npieces, G = fixup_group(np);
    const int g0 = (u.piece / G) * G, gn = min(G, np - g0), ngr = (np + G - 1) / G;
    const int64_t sb = u.slot_base;
    fixup_write<NJ, QPC, CSTRIDE>(acc, ws, sb + u.piece, npad, g, base, hoff);
    if (!arrive_last(ctr0 + (sb + g0) * cstride, gn, lane)) return;
    fixup_sum<NJ, QPC, CSTRIDE>(acc, ws, sb + g0, 1, gn, npad, g, base, hoff);
    if (ngr > 1) {
        fixup_write<NJ, QPC, CSTRIDE>(acc, ws, sb + g0, npad, g, base, hoff);
        if (!arrive_last(ctr0 + (sb + 1) * cstride, ngr, lane)) return;
        fixup_sum<NJ, QPC, CSTRIDE>(acc, ws, sb, G, ngr, npad, g, base, hoff);
    }
    store_tile<NJ, VEC, QPC, CSTRIDE>(C, ldc, M, N, u.wb, g, base, hoff, acc, false, rowmap);
}

// --------------------------------------------------- S1: A batch producer (one warp)
// Scatters the non-zeros of TC blocks [b0, b0+nb) into zeroed lane-major mma
// fragments (TF32-rounded) and copies their 8 B-row ids.
template <int DT>
__device__ __forceinline__ void produce_a_batch(int b0, int nb, const int32_t* __restrict__ tco,
                                                const uint8_t* __restrict__ lid, const int32_t* __restrict__ atob,
                                                const void* __restrict__ avals, uint32_t* fr, int32_t* ids,
                                                int32_t* s_tco, int lane) {
    constexpr int FW = Traits<DT>::FRAG_WORDS;
    if (lane < nb) s_tco[lane] = tco[b0 + lane];
    if (lane == 0) s_tco[nb] = tco[b0 + nb];
    for (int k = lane; k < 2 * nb; k += 32)
        reinterpret_cast<int4*>(ids)[k] = __ldg(reinterpret_cast<const int4*>(atob + (int64_t)b0 * 8) + k);
    for (int k = lane; k < nb * 32 * FW / 4; k += 32) reinterpret_cast<uint4*>(fr)[k] = make_uint4(0u, 0u, 0u, 0u);
    __syncwarp();
    const int e0 = s_tco[0], e1 = s_tco[nb];
    for (int base = e0; base < e1; base += 32 * 8) {
        int idv[8];
        uint32_t val[8];
#pragma unroll
        for (int q = 0; q < 8; ++q) {
            const int e = base + q * 32 + lane;
            if (e < e1) {
                idv[q] = lid[e];
                val[q] = (DT == DTC_TF32) ? __float_as_uint(__ldg(reinterpret_cast<const float*>(avals) + e))
                                          : (uint32_t)__ldg(reinterpret_cast<const unsigned short*>(avals) + e);
            }
        }
#pragma unroll
        for (int q = 0; q < 8; ++q) {
            const int e = base + q * 32 + lane;
            if (e < e1) {
                int lo = 0, hi = nb;  // block j of entry e: s_tco[j] <= e < s_tco[j+1]
                while (hi - lo > 1) {
                    const int mid = (lo + hi) >> 1;
                    if (s_tco[mid] <= e) lo = mid; else hi = mid;
                }
                uint32_t* f = fr + lo * 32 * FW;
                const int slot = frag_slot<DT>(idv[q]);
                if (DT == DTC_TF32) f[slot] = to_tf32(__uint_as_float(val[q]));
                else reinterpret_cast<unsigned short*>(f)[slot] = (unsigned short)val[q];
            }
        }
    }
    __syncwarp();
}

// ============================================================ main path: TMA gather4
// Column slice of a consumer warp = one 128-byte box column of B (32 fp32 / 64 fp16).
// Stage s of the B ring holds, for every active warp slice, 8 rows x 128 B
// (two gather4 boxes: rows 0-3 then rows 4-7) at ring + s*WARPS*1KB + warp*1KB,
// 128B-swizzled: 16-byte chunk c of row r sits at chunk c ^ r.
//  TF32: thread (g,t) reads rows t and t+4 at chunk cg = (g>>1) + 4*(g&1) -> the 8
//        lanes of an LDS.128 phase hit 8 distinct chunks (conflict-free); virtual mma
//        column g is actual column n0 + 4*cg + jj, so the thread ends up owning
//        columns n0 + 4t + [0,4) and n0 + 16 + 4t + [0,4).
//  FP16: thread (g,t) reads rows 2t and 2t+1 at chunk g (conflict-free), owning
//        columns n0 + 16t + [0,16) (as in the register-remap of P:313-319).
template <int DT, int WARPS, bool VEC>
__global__ void __launch_bounds__((WARPS + 2) * 32)
k_spmm_tma(const __grid_constant__ CUtensorMap bmap, const Unit* __restrict__ units, const int32_t* __restrict__ rwo,
           const int32_t* __restrict__ tco, const uint8_t* __restrict__ lid, const int32_t* __restrict__ atob,
           const void* __restrict__ avals, float* __restrict__ C, int64_t ldc, int64_t M, int64_t N,
           float* __restrict__ ws, int32_t* __restrict__ counters, int64_t npad,
           const int32_t* __restrict__ rowmap) {
    using Tr = Traits<DT>;
    constexpr int NJ = Tr::NJ, COLW = Tr::COLW, FW = Tr::FRAG_WORDS;
    constexpr int S = kChunk;
    constexpr int STAGE = WARPS * 1024;                   // bytes per B stage
    constexpr int R = kBRingBytes / STAGE > 16 ? 16 : kBRingBytes / STAGE;
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    // 1024-byte align the ring (128B swizzle atom)
    uint8_t* sbase = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    uint8_t* ring = sbase;                                                    // [R][STAGE]
    uint32_t* s_frag = reinterpret_cast<uint32_t*>(sbase + R * STAGE);        // [2][S][32*FW]
    int32_t* s_ids = reinterpret_cast<int32_t*>(s_frag + 2 * S * 32 * FW);    // [2][S][8]
    int32_t* s_tco = s_ids + 2 * S * 8;                                       // [S+1]
    __shared__ __align__(8) uint64_t bar_afull[2], bar_aempty[2], bar_bfull[R], bar_bempty[R];

    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const Unit u = units[blockIdx.x];
    const int64_t ncta0 = (int64_t)blockIdx.y * WARPS * COLW;
    const int64_t nact64 = (N - ncta0 + COLW - 1) / COLW;
    const int nact = nact64 < WARPS ? (int)nact64 : WARPS;
    const int nblocks = u.be - u.bb;
    const int nbatch = (nblocks + S - 1) / S;
    if (threadIdx.x == 0) {
        for (int i = 0; i < 2; ++i) {
            mbar_init(&bar_afull[i], 1);
            mbar_init(&bar_aempty[i], nact + 1);   // consumers + the B producer (reads ids)
        }
        for (int i = 0; i < R; ++i) {
            mbar_init(&bar_bfull[i], 1);
            mbar_init(&bar_bempty[i], nact);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();

    if (warp == WARPS) {
        // ================= A producer (S1) =================
        for (int c = 0; c < nbatch; ++c) {
            const int buf = c & 1;
            if (c >= 2) mbar_wait(&bar_aempty[buf], ((c >> 1) - 1) & 1);
            const int b0 = u.bb + c * S;
            produce_a_batch<DT>(b0, min(S, u.be - b0), tco, lid, atob, avals, s_frag + buf * S * 32 * FW,
                                s_ids + buf * S * 8, s_tco, lane);
            if (lane == 0) mbar_arrive(&bar_afull[buf]);
            __syncwarp();
        }
        return;
    }
    if (warp == WARPS + 1) {
        // ================= B producer (S2): gather4 into the swizzled ring =================
        const uint32_t bytes = (uint32_t)nact * 1024u;
        const int slice = lane >> 1, half = lane & 1;
        const int col = (int)(ncta0 + (int64_t)slice * COLW);
        for (int i = 0; i < nblocks; ++i) {
            const int c = i / S, j = i % S, s = i % R;
            if (j == 0) mbar_wait(&bar_afull[c & 1], (c >> 1) & 1);
            if (i >= R) mbar_wait(&bar_bempty[s], ((i / R) - 1) & 1);
            if (lane == 0) mbar_arrive_tx(&bar_bfull[s], bytes);
            if (slice < nact) {
                const int4 r = reinterpret_cast<const int4*>(s_ids + (c & 1) * S * 8 + j * 8)[half];
                const uint32_t dst = smem_u32(ring + s * STAGE + slice * 1024 + half * 512);
                asm volatile(
                    "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes"
                    " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(dst),
                    "l"(&bmap), "r"(col), "r"(r.x), "r"(r.y), "r"(r.z), "r"(r.w), "r"(smem_u32(&bar_bfull[s]))
                    : "memory");
            }
            if (j == S - 1 || i == nblocks - 1) {   // done reading this batch's ids
                __syncwarp();
                if (lane == 0) mbar_arrive(&bar_aempty[c & 1]);
            }
        }
        return;
    }
    if (warp >= nact) return;

    // ================= consumers (S3 mma, S4 epilogue) =================
    const int g = lane >> 2, t = lane & 3;
    const int64_t n0 = ncta0 + (int64_t)warp * COLW;
    const int64_t base = (DT == DTC_TF32) ? n0 + 4 * t : n0 + 16 * t;
    const int hoff = (DT == DTC_TF32) ? 16 : 8;
    const bool split = u.split_id >= 0;
    // smem byte offsets of this thread's two 16-byte B reads inside a warp slice
    int off0, off1;
    if (DT == DTC_TF32) {
        const int cg = (g >> 1) + 4 * (g & 1);
        off0 = t * 128 + ((cg ^ t) << 4);
        off1 = (t + 4) * 128 + ((cg ^ (t + 4)) << 4);
    } else {
        off0 = (2 * t) * 128 + ((g ^ (2 * t)) << 4);
        off1 = (2 * t + 1) * 128 + ((g ^ (2 * t + 1)) << 4);
    }
    const uint8_t* myring = ring + warp * 1024;

    float acc[NJ][4];
#pragma unroll
    for (int j = 0; j < NJ; ++j) acc[j][0] = acc[j][1] = acc[j][2] = acc[j][3] = 0.f;

    int64_t cur = u.wb;
    int64_t next_end = INT_MAX;
    if (!split) {
        while (cur < u.we && rwo[cur + 1] <= u.bb) { store_tile<NJ, VEC>(C, ldc, M, N, cur, g, base, hoff, acc, true, rowmap); ++cur; }
        next_end = cur < u.we ? rwo[cur + 1] : INT_MAX;
    }

    for (int i = 0; i < nblocks; ++i) {
        const int c = i / S, j = i % S, s = i % R;
        if (j == 0) mbar_wait(&bar_afull[c & 1], (c >> 1) & 1);
        mbar_wait(&bar_bfull[s], (i / R) & 1);
        const uint32_t* fr = s_frag + (c & 1) * S * 32 * FW + j * 32 * FW;
        const uint4 bv0 = *reinterpret_cast<const uint4*>(myring + s * STAGE + off0);
        const uint4 bv1 = *reinterpret_cast<const uint4*>(myring + s * STAGE + off1);
        if (DT == DTC_TF32) {
            const uint4 av = reinterpret_cast<const uint4*>(fr)[lane];
            const uint32_t a[4] = {av.x, av.y, av.z, av.w};
            const uint32_t x0[4] = {bv0.x, bv0.y, bv0.z, bv0.w};
            const uint32_t x1[4] = {bv1.x, bv1.y, bv1.z, bv1.w};
#pragma unroll
            for (int jj = 0; jj < NJ; ++jj)
                mma_tf32(acc[jj], a, x0[jj], x1[jj]);
        } else {
            const uint2 av = reinterpret_cast<const uint2*>(fr)[lane];
            const uint32_t a[2] = {av.x, av.y};
            const uint32_t x0[4] = {bv0.x, bv0.y, bv0.z, bv0.w};
            const uint32_t x1[4] = {bv1.x, bv1.y, bv1.z, bv1.w};
#pragma unroll
            for (int jj = 0; jj < NJ; ++jj) {
                const uint32_t bb = __byte_perm(x0[jj >> 1], x1[jj >> 1], (jj & 1) ? 0x7632 : 0x5410);
                mma_f16(acc[jj], a, bb);
            }
        }
        __syncwarp();
        if (lane == 0) {
            mbar_arrive(&bar_bempty[s]);
            if (j == S - 1 || i == nblocks - 1) mbar_arrive(&bar_aempty[c & 1]);
        }
        const int64_t b = u.bb + i;
        if (b + 1 == next_end) {   // S4: window boundary -> store and reset
            store_tile<NJ, VEC>(C, ldc, M, N, cur, g, base, hoff, acc, false, rowmap);
#pragma unroll
            for (int jj = 0; jj < NJ; ++jj) acc[jj][0] = acc[jj][1] = acc[jj][2] = acc[jj][3] = 0.f;
            ++cur;
            while (cur < u.we && rwo[cur + 1] == rwo[cur]) { store_tile<NJ, VEC>(C, ldc, M, N, cur, g, base, hoff, acc, true, rowmap); ++cur; }
            next_end = cur < u.we ? rwo[cur + 1] : INT_MAX;
        }
    }
    if (!split) {
        while (cur < u.we) { store_tile<NJ, VEC>(C, ldc, M, N, cur, g, base, hoff, acc, true, rowmap); ++cur; }
        return;
    }
    // S5: split-window fixup per consumer warp
    split_fixup<NJ, VEC>(u, acc, ws, npad, counters + blockIdx.y * 8 + warp, (int64_t)gridDim.y * 8, C, ldc, M, N, g,
                         lane, base, hoff, rowmap);
}

// ============================================================ fallback: register gather
// 64 zero bytes that padded (-1) B rows and columns beyond N read instead of B
// (branch-free gather: the address is selected, the load is unconditional).
__device__ __align__(128) uint4 g_zero_line[8];

// 16-byte read-only load of p if pred, else zeros -- branch-free (predicated LDG).
__device__ __forceinline__ V16 ldg16_pred(const void* p, bool pred) {
    V16 v;
    asm volatile(
        "{\n"
        ".reg .pred q;\n"
        "setp.ne.b32 q, %5, 0;\n"
        "mov.b32 %0, 0; mov.b32 %1, 0; mov.b32 %2, 0; mov.b32 %3, 0;\n"
        "@q ld.global.nc.v4.u32 {%0, %1, %2, %3}, [%4];\n"
        "}\n"
        : "=r"(v.w[0]), "=r"(v.w[1]), "=r"(v.w[2]), "=r"(v.w[3])
        : "l"(p), "r"((int)pred));
    return v;
}

template <int DT, bool VEC>
__device__ __forceinline__ V16 load_b(const void* __restrict__ B, int64_t ldb, int row, int64_t col, int64_t N) {
    using E = typename Traits<DT>::elt;
    const E* p = reinterpret_cast<const E*>(B) + (int64_t)row * ldb + col;
    if (VEC) return ldg16_pred(p, row >= 0 && col < N);
    V16 v;
    v.w[0] = v.w[1] = v.w[2] = v.w[3] = 0u;
    if (row < 0) return v;
    {
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

// All warps of the CTA share a double-buffered A pipeline over chunks of kChunk
// TC blocks: the global loads for chunk c+1's non-zeros and chunk c+2's offsets /
// B-row ids are issued into registers BEFORE chunk c is computed and only stored
// to smem at the chunk boundary, so FetchSparse never exposes memory latency
// (the paper's sparse double buffering, made two-deep).  Each warp
// streams its 32/64-column B slice with a kPrefetch-deep register ring that runs
// continuously across chunk boundaries (VFetchDense + remap).
// shared-memory bytes of the register-gather kernel (A chunks double buffered)
template <int DT, int W>
constexpr int ldg_smem_bytes() {
    constexpr int S = ldg_chunk<DT, W>();
    return 2 * S * 32 * Traits<DT>::FRAG_WORDS * 4 + 2 * S * 8 * 4 + 2 * (S + 1) * 4;
}

template <int DT, int WARPS, bool VEC, int CW>
__global__ void __launch_bounds__(WARPS * 32, ldg_min_blocks<DT, WARPS, CW>())
k_spmm_ldg(const Unit* __restrict__ units, const int32_t* __restrict__ rwo, const int32_t* __restrict__ tco,
           const uint8_t* __restrict__ lid, const int32_t* __restrict__ atob, const void* __restrict__ avals,
           const void* __restrict__ B, int64_t ldb, float* __restrict__ C, int64_t ldc, int64_t M, int64_t N,
           float* __restrict__ ws, int32_t* __restrict__ counters, int64_t npad,
           const int32_t* __restrict__ rowmap) {
    using Tr = Traits<DT>;
    constexpr int NJ1 = Tr::NJ, COLW1 = Tr::COLW, VW = Tr::VW, FW = Tr::FRAG_WORDS;
    constexpr int NJ = NJ1 * CW;          // n8 mmas per TC block per warp (CW column chunks)
    constexpr int COLW = COLW1 * CW;      // columns per warp
    constexpr int QPC = NJ1 / 4;          // accumulator quads per column chunk
    constexpr int P = ldg_prefetch<DT, WARPS>();
    constexpr int S = ldg_chunk<DT, WARPS>();
    constexpr int NT = WARPS * 32;
    constexpr int TPT = (S + 1 + NT - 1) / NT;      // TCOffset values per thread
    constexpr int IPT = (2 * S + NT - 1) / NT;      // int4 of B-row ids per thread
    constexpr int KE = 512 / NT < 1 ? 1 : (512 / NT > 4 ? 4 : 512 / NT);  // non-zeros per thread prefetched per chunk
    extern __shared__ __align__(16) uint32_t smem[];
    uint32_t* s_frag = smem;                                                 // [2][S][32*FW]
    int32_t* s_ids = reinterpret_cast<int32_t*>(smem + 2 * S * 32 * FW);     // [2][S][8]
    int32_t* s_tco = s_ids + 2 * S * 8;                                      // [2][S+1]

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int g = lane >> 2, t = lane & 3;
    const Unit u = units[blockIdx.x];
    const int64_t n0 = ((int64_t)blockIdx.y * WARPS + warp) * COLW;
    const bool active = n0 < N;
    const int64_t bcol = n0 + (int64_t)VW * g;
    const int64_t base = n0 + 2 * NJ1 * t;
    const int hoff = NJ1;
    const bool split = u.split_id >= 0;
    const int nblocks = u.be - u.bb;
    const int nchunks = (nblocks + S - 1) / S;
    auto chunk_nb = [&](int c) { return min(S, nblocks - c * S); };

    // ---- A pipeline pieces (register staging -> smem)
    int m_tco[TPT];
    int4 m_ids[IPT];
    auto meta_load = [&](int c) {
        const int nb = chunk_nb(c), b0 = u.bb + c * S;
#pragma unroll
        for (int k = 0; k < TPT; ++k) {
            const int x = tid + k * NT;
            if (x <= nb) m_tco[k] = tco[b0 + x];
        }
#pragma unroll
        for (int k = 0; k < IPT; ++k) {
            const int x = tid + k * NT;
            if (x < 2 * nb) m_ids[k] = __ldg(reinterpret_cast<const int4*>(atob + (int64_t)b0 * 8) + x);
        }
    };
    auto meta_store = [&](int c, int buf) {
        const int nb = chunk_nb(c);
#pragma unroll
        for (int k = 0; k < TPT; ++k) {
            const int x = tid + k * NT;
            if (x <= nb) s_tco[buf * (S + 1) + x] = m_tco[k];
        }
#pragma unroll
        for (int k = 0; k < IPT; ++k) {
            const int x = tid + k * NT;
            if (x < 2 * nb) {
                int4 v = m_ids[k];
                if (DT == DTC_TF32) {
                    // block row ids r0..r7 arrive as int4 {r0..r3}, {r4..r7}; store as
                    // r0 r4 r1 r5 r2 r6 r3 r7 so thread t reads (r_t, r_t+4) with one LDS.64
                    int* d = s_ids + buf * S * 8 + (x >> 1) * 8 + (x & 1);
                    d[0] = v.x; d[2] = v.y; d[4] = v.z; d[6] = v.w;
                } else {
                    reinterpret_cast<int4*>(s_ids + buf * S * 8)[x] = v;
                }
            }
        }
        uint4* fr = reinterpret_cast<uint4*>(s_frag + buf * S * 32 * FW);
        for (int x = tid; x < nb * 32 * FW / 4; x += NT) fr[x] = make_uint4(0u, 0u, 0u, 0u);
    };
    int e_id[KE];
    uint32_t e_val[KE];
    auto ent_val = [&](int e) -> uint32_t {
        return (DT == DTC_TF32) ? __float_as_uint(__ldg(reinterpret_cast<const float*>(avals) + e))
                                : (uint32_t)__ldg(reinterpret_cast<const unsigned short*>(avals) + e);
    };
    auto ent_load_n = [&](int buf, int nb) {
        const int e0 = s_tco[buf * (S + 1)], e1 = s_tco[buf * (S + 1) + nb];
#pragma unroll
        for (int k = 0; k < KE; ++k) {
            const int e = e0 + tid + k * NT;
            if (e < e1) {
                e_id[k] = lid[e];
                e_val[k] = ent_val(e);
            }
        }
    };
    auto put = [&](int buf, int nb, int e, int id, uint32_t v) {
        const int32_t* tc = s_tco + buf * (S + 1);
        int lo = 0, hi = nb;   // block j of entry e: tc[j] <= e < tc[j+1]
        while (hi - lo > 1) {
            const int mid = (lo + hi) >> 1;
            if (tc[mid] <= e) lo = mid; else hi = mid;
        }
        uint32_t* f = s_frag + buf * S * 32 * FW + lo * 32 * FW;
        const int slot = frag_slot<DT>(id);
        if (DT == DTC_TF32) f[slot] = to_tf32(__uint_as_float(v));
        else reinterpret_cast<unsigned short*>(f)[slot] = (unsigned short)v;
    };
    auto ent_store_n = [&](int buf, int nb) {
        const int e0 = s_tco[buf * (S + 1)], e1 = s_tco[buf * (S + 1) + nb];
#pragma unroll
        for (int k = 0; k < KE; ++k) {
            const int e = e0 + tid + k * NT;
            if (e < e1) put(buf, nb, e, e_id[k], e_val[k]);
        }
        for (int e = e0 + KE * NT + tid; e < e1; e += NT) put(buf, nb, e, lid[e], ent_val(e));  // dense chunks
    };

    float acc[NJ][4];
#pragma unroll
    for (int j = 0; j < NJ; ++j) acc[j][0] = acc[j][1] = acc[j][2] = acc[j][3] = 0.f;

    int cur = u.wb;          // window cursor (int32: W, T < 2^31)
    int next_end = INT_MAX;
    if (!split) {
        while (cur < u.we && rwo[cur + 1] <= u.bb) {
            if (active) store_tile<NJ, VEC, QPC, COLW1>(C, ldc, M, N, cur, g, base, hoff, acc, true, rowmap);
            ++cur;
        }
        next_end = cur < u.we ? rwo[cur + 1] : INT_MAX;
    }

    if (nchunks > 0) {
        // prologue: chunks 0 and 1 staged, chunk 1's non-zeros and chunk 2's meta in flight
        meta_load(0);
        meta_store(0, 0);
        if (nchunks > 1) { meta_load(1); meta_store(1, 1); }
        __syncthreads();
        ent_load_n(0, chunk_nb(0));
        ent_store_n(0, chunk_nb(0));
        __syncthreads();
        if (nchunks > 1) ent_load_n(1, chunk_nb(1));
        if (nchunks > 2) meta_load(2);

        {
        V16 b0[P][CW], b1[P][CW];
        // thread's two B rows of block i: TF32 (t, t+4), FP16 (2t, 2t+1) -> adjacent id slots 2t, 2t+1
        auto ids_of = [&](int i) -> int2 {
            return *reinterpret_cast<const int2*>(s_ids + ((i / S) & 1) * S * 8 + (i % S) * 8 + 2 * t);
        };
        // VEC: byte pointer of this thread's 16-byte column vector in B row 0; padded rows and
        // columns >= N are redirected to the zero line (no predication, no divergence)
        const char* bthr = reinterpret_cast<const char*>(B) + bcol * (int64_t)sizeof(typename Tr::elt);
        const uint64_t ldb_bytes = (uint64_t)ldb * sizeof(typename Tr::elt);
#if defined(DTC_L2_HINTS) && (DTC_L2_HINTS & 1)
        const uint64_t pol_b = l2_policy_last();
#endif
        auto gather = [&](int row, int cw) -> V16 {
            if (VEC) {
                const bool ok = row >= 0 && (bcol + cw * COLW1) < N;
                const char* p = ok ? bthr + (uint64_t)(uint32_t)row * ldb_bytes + cw * COLW1 * (int)sizeof(typename Tr::elt)
                                   : reinterpret_cast<const char*>(g_zero_line);
#if defined(DTC_L2_HINTS) && (DTC_L2_HINTS & 1)
                const uint4 x = ldg_hint(p, pol_b);
#else
                const uint4 x = __ldg(reinterpret_cast<const uint4*>(p));
#endif
                V16 v;
                v.w[0] = x.x; v.w[1] = x.y; v.w[2] = x.z; v.w[3] = x.w;
                return v;
            }
            return load_b<DT, VEC>(B, ldb, row, bcol + cw * COLW1, N);
        };
        if (active) {
#pragma unroll
            for (int q = 0; q < P; ++q) {
                if (q < nblocks) {
                    const int2 id = ids_of(q);
#pragma unroll
                    for (int cw = 0; cw < CW; ++cw) {
                        b0[q][cw] = gather(id.x, cw);
                        b1[q][cw] = gather(id.y, cw);
                    }
                }
            }
        }
        for (int i0 = 0; i0 < nblocks; i0 += P) {
#pragma unroll
            for (int q = 0; q < P; ++q) {
                const int i = i0 + q;
                if (i < nblocks) {
                    const int c = i / S, j = i % S;
                    if (active) {
                        const uint32_t* fr = s_frag + (c & 1) * S * 32 * FW + j * 32 * FW;
                        if (DT == DTC_TF32) {
                            const uint4 av = reinterpret_cast<const uint4*>(fr)[lane];
                            const uint32_t a[4] = {av.x, av.y, av.z, av.w};
#pragma unroll
                            for (int cw = 0; cw < CW; ++cw)
#pragma unroll
                                for (int jj = 0; jj < NJ1; ++jj)
                                    mma_tf32(acc[cw * NJ1 + jj], a, b0[q][cw].w[jj], b1[q][cw].w[jj]);
                        } else {
                            const uint2 av = reinterpret_cast<const uint2*>(fr)[lane];
                            const uint32_t a[2] = {av.x, av.y};
#pragma unroll
                            for (int cw = 0; cw < CW; ++cw)
#pragma unroll
                                for (int jj = 0; jj < NJ1; ++jj) {
                                    const uint32_t bb = __byte_perm(b0[q][cw].w[jj >> 1], b1[q][cw].w[jj >> 1],
                                                                    (jj & 1) ? 0x7632 : 0x5410);
                                    mma_f16(acc[cw * NJ1 + jj], a, bb);
                                }
                        }
                        if (i + P < nblocks) {
                            const int2 id = ids_of(i + P);
#pragma unroll
                            for (int cw = 0; cw < CW; ++cw) {
                                b0[q][cw] = gather(id.x, cw);
                                b1[q][cw] = gather(id.y, cw);
                            }
                        }
                        if (u.bb + i + 1 == next_end) {
                            store_tile<NJ, VEC, QPC, COLW1>(C, ldc, M, N, cur, g, base, hoff, acc, false, rowmap);
#pragma unroll
                            for (int jj = 0; jj < NJ; ++jj) acc[jj][0] = acc[jj][1] = acc[jj][2] = acc[jj][3] = 0.f;
                            ++cur;
                            while (cur < u.we && rwo[cur + 1] == rwo[cur]) {
                                store_tile<NJ, VEC, QPC, COLW1>(C, ldc, M, N, cur, g, base, hoff, acc, true, rowmap);
                                ++cur;
                            }
                            next_end = cur < u.we ? rwo[cur + 1] : INT_MAX;
                        }
                    }
                }
            }
            const int nxt = i0 + P;   // S is a multiple of P: chunk boundaries fall between groups
            if (nxt % S == 0 && nxt < nblocks) {
                // chunk boundary (CTA-uniform): finish chunk c+1's fragments, recycle buffer c&1
                const int c = nxt / S - 1;
                ent_store_n((c + 1) & 1, chunk_nb(c + 1));
                __syncthreads();
                if (c + 2 < nchunks) meta_store(c + 2, c & 1);
                __syncthreads();
                if (c + 2 < nchunks) ent_load_n(c & 1, chunk_nb(c + 2));
                if (c + 3 < nchunks) meta_load(c + 3);
            }
        }
        }
    }
    if (!active) return;
    if (!split) {
        while (cur < u.we) { store_tile<NJ, VEC, QPC, COLW1>(C, ldc, M, N, cur, g, base, hoff, acc, true, rowmap); ++cur; }
        return;
    }
    split_fixup<NJ, VEC, QPC, COLW1>(u, acc, ws, npad, counters + blockIdx.y * 8 + warp, (int64_t)gridDim.y * 8, C,
                                     ldc, M, N, g, lane, base, hoff, rowmap);
}

// ============================================================ direct path (no shared memory)
// Every warp builds its own A fragment straight from ME-TCF + the occupancy mask, so there
// is no FetchSparse producer, no shared-memory scatter and no CTA barrier at all:
//  * k permutation: lane (g,t) takes B rows SparseAtoB[8b+2t] and [8b+2t+1] as its mma rows
//    k=t and k=t+4 (one 8-byte load).  The A columns are permuted the same way, so the
//    lane's four A slots are local ids 8g+2t, 8g+2t+1, 8(g+8)+2t, 8(g+8)+2t+1 -- the same
//    four slots in TF32 (a0,a2 | a1,a3) and FP16 (reg0 | reg1) fragment order.
//  * the value of slot id is TCValues[TCOffset[b] + popcount(mask[b] below id)] (C5), loaded
//    predicated on the mask bit; TF32 rounds it with cvt.rna once per block.
//  * a P-deep register pipeline per warp: block i+P's B rows and A values are issued right
//    after block i's mma, block i+2P's (ids, mask, TCOffset) one stage earlier.
template <int DT>
struct DirMeta {
    int2 ids;
    uint4 m;
    int base;
};

template <int DT, int WARPS, int CW, int PD>
constexpr int dir_maxregs() {
#if defined(DTC_DIR_MAXREGS) && defined(DTC_DIR_MAXREGS_H)
    return DT == DTC_FP16 ? DTC_DIR_MAXREGS_H : DTC_DIR_MAXREGS;
#else
    return DT == DTC_FP16 ? (PD == 1 ? 128 : 168) : (PD == 1 ? 96 : 128);
#endif
}
template <int DT, int WARPS, int CW, int PD>
constexpr int dir_min_blocks() {
    constexpr int b = 65536 / (WARPS * 32 * dir_maxregs<DT, WARPS, CW, PD>());
    return b > 32 ? 32 : (b < 1 ? 1 : b);
}
template <int DT>
constexpr int dir_depth() {
#ifdef DTC_DIR_DEPTH
    return DTC_DIR_DEPTH;
#else
    return 1;
#endif
}

__device__ __forceinline__ uint32_t ldg_u32_pred(const uint32_t* p, bool pred) {
    uint32_t v;
    asm volatile(
        "{\n"
        ".reg .pred q;\n"
        "setp.ne.b32 q, %2, 0;\n"
        "mov.b32 %0, 0;\n"
        "@q ld.global.nc.u32 %0, [%1];\n"
        "}\n"
        : "=r"(v)
        : "l"(p), "r"((int)pred));
    return v;
}
__device__ __forceinline__ uint32_t ldg_u16_pred(const unsigned short* p, bool pred) {
    unsigned short v;
    asm volatile(
        "{\n"
        ".reg .pred q;\n"
        "setp.ne.b32 q, %2, 0;\n"
        "mov.b16 %0, 0;\n"
        "@q ld.global.nc.u16 %0, [%1];\n"
        "}\n"
        : "=h"(v)
        : "l"(p), "r"((int)pred));
    return (uint32_t)v;
}

// (ids, mask, TCOffset) of TC block b for lane t: B rows SparseAtoB[8b+2t], [8b+2t+1]
template <int DT>
__device__ __forceinline__ DirMeta<DT> dir_load_meta(int b, int t, const int32_t* __restrict__ atob,
                                                     const uint4* __restrict__ mask, const int32_t* __restrict__ tco) {
    DirMeta<DT> mt;
    mt.ids = __ldg(reinterpret_cast<const int2*>(atob + (int64_t)b * 8) + t);
    mt.m = __ldg(mask + b);
    mt.base = __ldg(tco + b);
    return mt;
}
// A fragment of one TC block for lane (g,t) under the k permutation (slots 8g+2t, 8g+2t+1,
// 8(g+8)+2t, 8(g+8)+2t+1): value rank = popcount of the mask below the slot (C5)
template <int DT>
__device__ __forceinline__ void dir_load_a(const DirMeta<DT>& mt, uint32_t (&a)[Traits<DT>::FRAG_WORDS], int pos,
                                           uint32_t below, bool upper, const void* __restrict__ avals) {
    const uint32_t wl = upper ? mt.m.y : mt.m.x;
    const uint32_t wh = upper ? mt.m.w : mt.m.z;
    const int c0 = __popc(mt.m.x), c01 = c0 + __popc(mt.m.y);
    const int rl = mt.base + (upper ? c0 : 0) + __popc(wl & below);
    const int rh = mt.base + c01 + (upper ? __popc(mt.m.z) : 0) + __popc(wh & below);
    const bool p00 = (wl >> pos) & 1u, p01 = (wl >> (pos + 1)) & 1u;
    const bool p10 = (wh >> pos) & 1u, p11 = (wh >> (pos + 1)) & 1u;
    if (DT == DTC_TF32) {
        const uint32_t* v = reinterpret_cast<const uint32_t*>(avals);
        a[0] = to_tf32(__uint_as_float(ldg_u32_pred(v + rl, p00)));        // (g,   k=t)   id 8g+2t
        a[1] = to_tf32(__uint_as_float(ldg_u32_pred(v + rh, p10)));        // (g+8, k=t)
        a[2] = to_tf32(__uint_as_float(ldg_u32_pred(v + rl + p00, p01)));  // (g,   k=t+4) id 8g+2t+1
        a[3] = to_tf32(__uint_as_float(ldg_u32_pred(v + rh + p10, p11)));  // (g+8, k=t+4)
    } else {
        const unsigned short* v = reinterpret_cast<const unsigned short*>(avals);
        a[0] = ldg_u16_pred(v + rl, p00) | (ldg_u16_pred(v + rl + p00, p01) << 16);   // (g, 2t), (g, 2t+1)
        a[1] = ldg_u16_pred(v + rh, p10) | (ldg_u16_pred(v + rh + p10, p11) << 16);   // (g+8, ...)
    }
}

template <int DT, int WARPS, bool VEC, int CW, int PD>
__global__ void __launch_bounds__(WARPS * 32, dir_min_blocks<DT, WARPS, CW, PD>())
k_spmm_dir(const Unit* __restrict__ units, const int32_t* __restrict__ rwo, const int32_t* __restrict__ tco,
           const uint4* __restrict__ mask, const int32_t* __restrict__ atob, const void* __restrict__ avals,
           const void* __restrict__ B, int64_t ldb, float* __restrict__ C, int64_t ldc, int64_t M, int64_t N,
           float* __restrict__ ws, int32_t* __restrict__ counters, int64_t npad,
           const int32_t* __restrict__ rowmap, int num_units, int nws, int pass_ws) {
    using Tr = Traits<DT>;
    constexpr int NJ1 = Tr::NJ, COLW1 = Tr::COLW, VW = Tr::VW, FW = Tr::FRAG_WORDS;
    constexpr int NJ = NJ1 * CW;
    constexpr int COLW = COLW1 * CW;
    constexpr int QPC = NJ1 / 4;
    using E = typename Tr::elt;

    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int g = lane >> 2, t = lane & 3;
    // work item = (unit, warp slice of COLW columns); warps are independent (no CTA barrier).
    // Items run in passes of pass_ws slices (a pass's B columns sized to stay L2-resident),
    // unit-major inside a pass so the slices of one unit land on neighbouring warps.
    const int64_t item = (int64_t)blockIdx.x * WARPS + warp;
    const int64_t per = (int64_t)num_units * pass_ws;
    const int p = (int)(item / per);
    const int64_t r = item - (int64_t)p * per;
    const int pw = min(pass_ws, nws - p * pass_ws);
    if (pw <= 0) return;
    const int wsl = p * pass_ws + (int)(r % pw);
    const int64_t n0 = (int64_t)wsl * COLW;
    const Unit u = units[r / pw];
    const int64_t bcol = n0 + (int64_t)VW * g;
    const int64_t base = n0 + 2 * NJ1 * t;
    const int hoff = NJ1;
    const bool split = u.split_id >= 0;
    const int nblocks = u.be - u.bb;

    // this lane's mask bits: slots (8g+2t, +1) in word g>>2, (64+8g+2t, +1) in word 2+(g>>2)
    const int pos = 8 * (g & 3) + 2 * t;
    const uint32_t below = (1u << pos) - 1u;
    const bool upper = g >= 4;

    auto load_meta = [&](int b) -> DirMeta<DT> { return dir_load_meta<DT>(b, t, atob, mask, tco); };
    auto load_a = [&](const DirMeta<DT>& mt, uint32_t (&a)[FW]) { dir_load_a<DT>(mt, a, pos, below, upper, avals); };
    const char* bthr = reinterpret_cast<const char*>(B) + bcol * (int64_t)sizeof(E);
    const uint64_t ldb_bytes = (uint64_t)ldb * sizeof(E);
    auto gather = [&](int row, int cw) -> V16 {
        if (VEC) {
            const bool ok = row >= 0 && (bcol + cw * COLW1) < N;
            const char* p = ok ? bthr + (uint64_t)(uint32_t)row * ldb_bytes + cw * COLW1 * (int)sizeof(E)
                               : reinterpret_cast<const char*>(g_zero_line);
            const uint4 x = __ldg(reinterpret_cast<const uint4*>(p));
            V16 v;
            v.w[0] = x.x; v.w[1] = x.y; v.w[2] = x.z; v.w[3] = x.w;
            return v;
        }
        return load_b<DT, VEC>(B, ldb, row, bcol + cw * COLW1, N);
    };

    float acc[NJ][4];
#pragma unroll
    for (int j = 0; j < NJ; ++j) acc[j][0] = acc[j][1] = acc[j][2] = acc[j][3] = 0.f;

    int cur = u.wb;
    int next_end = INT_MAX;
    if (!split) {
        while (cur < u.we && rwo[cur + 1] <= u.bb) {
            store_tile<NJ, VEC, QPC, COLW1>(C, ldc, M, N, cur, g, base, hoff, acc, true, rowmap);
            ++cur;
        }
        next_end = cur < u.we ? rwo[cur + 1] : INT_MAX;
    }

    DirMeta<DT> mt[PD];
    uint32_t af[PD][FW];
    V16 b0[PD][CW], b1[PD][CW];
    auto issue = [&](int q) {
#pragma unroll
        for (int cw = 0; cw < CW; ++cw) {
            b0[q][cw] = gather(mt[q].ids.x, cw);
            b1[q][cw] = gather(mt[q].ids.y, cw);
        }
        load_a(mt[q], af[q]);
    };
#pragma unroll
    for (int q = 0; q < PD; ++q)
        if (q < nblocks) mt[q] = load_meta(u.bb + q);
#pragma unroll
    for (int q = 0; q < PD; ++q)
        if (q < nblocks) {
            issue(q);
            if (q + PD < nblocks) mt[q] = load_meta(u.bb + q + PD);
        }
    for (int i0 = 0; i0 < nblocks; i0 += PD) {
#pragma unroll
        for (int q = 0; q < PD; ++q) {
            const int i = i0 + q;
            if (i < nblocks) {
                if (DT == DTC_TF32) {
                    const uint32_t a[4] = {af[q][0], af[q][1], af[q][2], af[q][3]};
#pragma unroll
                    for (int cw = 0; cw < CW; ++cw)
#pragma unroll
                        for (int jj = 0; jj < NJ1; ++jj)
                            mma_tf32(acc[cw * NJ1 + jj], a, b0[q][cw].w[jj], b1[q][cw].w[jj]);
                } else {
                    const uint32_t a[2] = {af[q][0], af[q][1]};
#pragma unroll
                    for (int cw = 0; cw < CW; ++cw)
#pragma unroll
                        for (int jj = 0; jj < NJ1; ++jj) {
                            const uint32_t bb = __byte_perm(b0[q][cw].w[jj >> 1], b1[q][cw].w[jj >> 1],
                                                            (jj & 1) ? 0x7632 : 0x5410);
                            mma_f16(acc[cw * NJ1 + jj], a, bb);
                        }
                }
                if (i + PD < nblocks) {
                    issue(q);
                    if (i + 2 * PD < nblocks) mt[q] = load_meta(u.bb + i + 2 * PD);
                }
                if (u.bb + i + 1 == next_end) {
                    store_tile<NJ, VEC, QPC, COLW1>(C, ldc, M, N, cur, g, base, hoff, acc, false, rowmap);
#pragma unroll
                    for (int jj = 0; jj < NJ; ++jj) acc[jj][0] = acc[jj][1] = acc[jj][2] = acc[jj][3] = 0.f;
                    ++cur;
                    while (cur < u.we && rwo[cur + 1] == rwo[cur]) {
                        store_tile<NJ, VEC, QPC, COLW1>(C, ldc, M, N, cur, g, base, hoff, acc, true, rowmap);
                        ++cur;
                    }
                    next_end = cur < u.we ? rwo[cur + 1] : INT_MAX;
                }
            }
        }
    }
    if (!split) {
        while (cur < u.we) { store_tile<NJ, VEC, QPC, COLW1>(C, ldc, M, N, cur, g, base, hoff, acc, true, rowmap); ++cur; }
        return;
    }
    split_fixup<NJ, VEC, QPC, COLW1>(u, acc, ws, npad, counters + wsl, (int64_t)nws, C, ldc, M, N, g, lane, base, hoff,
                                     rowmap);
}

// ============================================================ TMA path with padded rows (path 4)
// B rows arrive by TMA tile::gather4 in boxes of one 512-byte column slice plus 16 bytes of
// padding (128 fp32 / 256 fp16 columns + 4 / 8 extra), so the 4 rows of one gather4 sit 528
// bytes apart: 528 = 16 (mod 128) shifts each row by one 16-byte bank group.  One op gathers
// the block's even rows (SparseAtoB[0,2,4,6]) at slice offset 0, a second the odd rows at
// offset 2176 (TMA destinations are 128-byte aligned); lane (g,t) reads even row t and odd row
// t -- its mma rows k=t / k=t+4 (TF32, k permutation as k_spmm_dir) or k=2t / 2t+1 (FP16) --
// at 16-byte chunk c(g) = (g>>1) + 4(g&1) of a 128-byte segment, so the 8 lanes of an LDS.128
// phase hit 8 distinct bank groups: conflict-free without a swizzle, and 4x fewer TMA ops per
// byte than 128-byte swizzled boxes (the r01 gather4 ablation was op-rate bound).  The gather
// moves no data through the LSU pipe (the register gather's limiter: ncu l1tex data-pipe 85%);
// one producer warp runs up to pad_stages blocks ahead.  Consumer warps: 2 per slice, each
// owning 2 x 128-byte segments (64 fp32 / 128 fp16 columns); A fragments are built in
// registers from the occupancy mask one block ahead (as k_spmm_dir).
// Column ownership (virtual mma column v <-> chunk c(v)): TF32 thread holds columns
// seg + 4t + [0,4) and seg + 16 + 4t + [0,4); FP16 seg + 8t + [0,8) and seg + 32 + 8t + [0,8).
// Slice geometry, SEG = 128-byte segments per slice row: 4 (512-byte slices, 4-byte TMA
// elements, box 132) or 8 (1 KB slices, 8-byte TMA elements, box 130 -- one gather4 op moves
// 2x the bytes, for B rows of >= 1 KB).  Row pitch SEG*128 + 16 (= 16 mod 128).
template <int SEG> constexpr int pad_row_bytes() { return SEG * 128 + 16; }
template <int SEG> constexpr int pad_odd_off() { return (4 * pad_row_bytes<SEG>() + 127) / 128 * 128; }
template <int SEG> constexpr int pad_slice_bytes() { return (pad_odd_off<SEG>() + 4 * pad_row_bytes<SEG>() + 127) / 128 * 128; }
template <int SEG> constexpr int pad_tx_bytes() { return 8 * pad_row_bytes<SEG>(); }
static_assert(pad_row_bytes<4>() % 128 == 16 && pad_row_bytes<8>() % 128 == 16, "row pitch must be 16 mod 128");
static_assert(pad_row_bytes<2>() % 128 == 16 && pad_row_bytes<2>() % 8 == 0 && pad_row_bytes<4>() % 8 == 0 &&
                  pad_row_bytes<8>() % 8 == 0, "row pitch must be 16 mod 128 and whole 8-byte elements");
template <int SL>
constexpr int pad_stages() {
#ifdef DTC_PAD_STAGES
    return DTC_PAD_STAGES;
#else
    return SL == 1 ? 4 : (SL == 2 ? 4 : 3);
#endif
}
// A side of the TMA path: per batch of kPadBatch TC blocks, one bulk copy of the (16-byte
// aligned superset of the) batch's TCValues -- contiguous, TCOffset[b0] .. TCOffset[b0+16] --
// and one of its 16 occupancy masks, double buffered.
#ifndef DTC_PAD_BATCH
#define DTC_PAD_BATCH 16
#endif
constexpr int kPadBatch = DTC_PAD_BATCH;
// per-unit side record for the first batch (default on; DTC_PAD_FIRST=0 disables): kPadBatch x 8 SparseAtoB ids
// (-1 past the unit), TCOffset[bb], TCOffset[bb + min(kPadBatch, nb)], end of the first window, pad
constexpr int kFirstRec = kPadBatch * 8 + 4;
static_assert((kFirstRec * 4) % 16 == 0, "int4 loads of the side record");
constexpr int kPadAValBytes = kPadBatch * 512 + 128;       // >= batch x 128 values x 4 B + 16, 128-aligned
constexpr int kPadAIdsOff = kPadAValBytes + kPadBatch * 16;  // + one 16-byte mask per block
constexpr int kPadASlot = kPadAIdsOff + kPadBatch * 32;      // + 8 SparseAtoB ids per block (hybrid LDG warps)
static_assert(kPadBatch >= 1 && kPadBatch <= 16, "batch: the producer's lane pairs hold one block each");
template <int SL, int SEG>
constexpr size_t pad_smem_bytes_() { return (size_t)pad_stages<SL>() * SL * pad_slice_bytes<SEG>() + 2 * kPadASlot + 128; }
template <int SL, int SEG>
constexpr size_t pad_smem_bytes() { return pad_smem_bytes_<SL, SEG>(); }
template <int DT, int SL>
constexpr int pad_maxregs() {
#ifdef DTC_PAD_MAXREGS
    return DTC_PAD_MAXREGS;
#else
    return DT == DTC_FP16 ? 128 : 104;
#endif
}

__device__ __forceinline__ int64_t gtimer() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return (int64_t)t;
}
__device__ __forceinline__ int smid() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
    return (int)r;
}
__device__ __forceinline__ uint2 lds64(uint32_t a) {
    uint2 v;
    asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "r"(a));
    return v;
}
__device__ __forceinline__ uint4 lds128(uint32_t a) {
    uint4 v;
    asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
    return v;
}
__device__ __forceinline__ uint32_t lds32_pred(uint32_t a, bool p) {
    uint32_t v;
    asm volatile("{\n.reg .pred q;\nsetp.ne.b32 q, %2, 0;\nmov.b32 %0, 0;\n@q ld.shared.u32 %0, [%1];\n}\n"
                 : "=r"(v) : "r"(a), "r"((int)p));
    return v;
}
__device__ __forceinline__ uint32_t lds16_pred(uint32_t a, bool p) {
    unsigned short v;
    asm volatile("{\n.reg .pred q;\nsetp.ne.b32 q, %2, 0;\nmov.b16 %0, 0;\n@q ld.shared.u16 %0, [%1];\n}\n"
                 : "=h"(v) : "r"(a), "r"((int)p));
    return (uint32_t)v;
}

template <int DT, int SL, int SEG, int NL, bool VEC>
__global__ void __launch_bounds__((SL * SEG / 2 + NL + 1) * 32,
                                  65536 / ((SL * SEG / 2 + NL + 1) * 32 * pad_maxregs<DT, SL>()))
k_spmm_pad(const __grid_constant__ CUtensorMap bmap, const Unit* __restrict__ units, const int32_t* __restrict__ rwo,
           const int32_t* __restrict__ tco, const uint4* __restrict__ mask, const int32_t* __restrict__ atob,
           const void* __restrict__ avals, float* __restrict__ C, int64_t ldc, int64_t M, int64_t N,
           float* __restrict__ ws, int32_t* __restrict__ counters, int64_t npad,
           const int32_t* __restrict__ rowmap, int64_t* __restrict__ trace, const void* __restrict__ B,
           int64_t ldb, int num_units, int32_t* __restrict__ uctr, int te, int lsur,
           const int32_t* __restrict__ ufirst) {
    using Tr = Traits<DT>;
    constexpr int NJ1 = Tr::NJ, COLW1 = Tr::COLW, FW = Tr::FRAG_WORDS;
    constexpr int ELT = (int)sizeof(typename Tr::elt);
    // optional per-CTA timeline (dtc_set_trace): {cta, smid, t_start, t_first_issue, t_first_data,
    // t_consumer_done, nblocks, t_producer_done} in %globaltimer ns
    int64_t* tr = trace ? trace + ((int64_t)blockIdx.y * gridDim.x + blockIdx.x) * 8 : nullptr;
    if (tr && threadIdx.x == 0) {
        tr[0] = (int64_t)blockIdx.y * gridDim.x + blockIdx.x;
        tr[1] = smid();
        tr[2] = gtimer();
    }
    constexpr int CW = 2;                      // 128-byte segments per consumer warp
    constexpr int NJ = NJ1 * CW, QPC = NJ1 / 4;   // QPC quads per segment, segments COLW1 apart
    constexpr int R = pad_stages<SL>();
    constexpr int WPS = SEG / 2;               // consumer warps per slice
    constexpr int ROWB = pad_row_bytes<SEG>(), ODD = pad_odd_off<SEG>(), SLB = pad_slice_bytes<SEG>();
    constexpr int STAGE = SL * SLB;
    constexpr int SLICE_COLS = SEG * COLW1;    // 128 / 256 fp32 or 256 / 512 fp16 columns per slice
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    const uint32_t ring = (smem_u32(smem_raw) + 127u) & ~127u;       // [R][STAGE] B stages
    const uint32_t aring = ring + R * STAGE;                          // [2][kPadASlot] A batches
    __shared__ __align__(8) uint64_t bar_full[R], bar_empty[R], bar_afull[2], bar_aempty[2], bar_ufull[2], bar_uempty[2];
    __shared__ int s_abyte[2];   // byte offset of the batch's first value inside its A slot
    __shared__ int s_unit[2][10];   // published unit: Unit record, end block of its first window, index (-1 = done)

    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    // Units of this CTA: blockIdx.x only (one CTA per unit), or -- persistent launch -- the units
    // the producer draws from the column group's atomic counter uctr[2*blockIdx.y] (dynamic
    // balance; the last CTA resets it), or blockIdx.x + k*gridDim.x when uctr is null.  The
    // producer publishes each unit (record + end of its first window) to the consumers through
    // s_unit / bar_ufull / bar_uempty; the B ring and the A batches run on CTA-wide counters
    // (gi0 blocks, gc0 batches before the current unit), so prefetching continues across units.
    // CTA columns: SL TMA slices, then NL register-gather (LSU) warps of CW segments each (hybrid:
    // the TMA engine and the LSU pipe gather different columns of the same TC blocks concurrently)
    constexpr int CTA_COLS = SL * SLICE_COLS + NL * CW * COLW1;
    constexpr int WT = SL * WPS;               // TMA consumer warps
    const int64_t col0 = (int64_t)blockIdx.y * CTA_COLS;               // first C column of the CTA
    const int64_t nsl64 = (N - col0 + SLICE_COLS - 1) / SLICE_COLS;
    const int nsl = nsl64 < SL ? (int)(nsl64 > 0 ? nsl64 : 0) : SL;
    const int ncons = WPS * nsl;               // B-stage consumers
    const int nacons = ncons + NL;             // A-batch consumers
    if (threadIdx.x == 0) {
        for (int i = 0; i < R; ++i) {
            mbar_init(&bar_full[i], 1);
            mbar_init(&bar_empty[i], ncons);
        }
        for (int i = 0; i < 2; ++i) {
            mbar_init(&bar_afull[i], 1);
            mbar_init(&bar_aempty[i], nacons);
            mbar_init(&bar_ufull[i], 1);
            mbar_init(&bar_uempty[i], ncons);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();

    if (warp == WT + NL) {
        // ================= producer: A batches (bulk copies) + B gather4 (4 rows x one slice per op)
        const uint32_t tx = (uint32_t)nsl * pad_tx_bytes<SEG>();
        const int half = lane & 1, jl = lane >> 1;     // lane pair (2j, 2j+1): even / odd rows of block i0 + j
        const int32_t tcol = (int32_t)(col0 * ELT / te);  // TMA columns (te = 4- or 8-byte elements)
        const int32_t tslice = SEG * 128 / te;             // TMA columns per slice
        // Batch metadata is loaded one batch ahead -- across unit boundaries, with the next unit's
        // record loaded one unit ahead -- and only shuffled into gather4 row order when its batch
        // starts, so no load latency sits between two batches (or two units) of TMA issues.
        struct Raw { int4 mine; int e0, e1; };
        struct BatchMeta { int4 ids; int e0, e1; };
        auto load_raw = [&](const Unit& uu, int i0) -> Raw {
            Raw r;
            const int nbu = uu.be - uu.bb, i = i0 + jl;
            r.mine = i < nbu ? __ldg(reinterpret_cast<const int4*>(atob + (int64_t)(uu.bb + i) * 8) + half)
                             : make_int4(-1, -1, -1, -1);
            r.e0 = r.e1 = 0;
            if (lane == 0 && i0 < nbu) {
                r.e0 = __ldg(tco + uu.bb + i0);
                r.e1 = __ldg(tco + uu.bb + min(i0 + kPadBatch, nbu));
            }
            return r;
        };
        auto finish = [&](const Raw& r) -> BatchMeta {
            BatchMeta bm;
            int4 o;   // partner's half
            o.x = __shfl_xor_sync(0xffffffffu, r.mine.x, 1);
            o.y = __shfl_xor_sync(0xffffffffu, r.mine.y, 1);
            o.z = __shfl_xor_sync(0xffffffffu, r.mine.z, 1);
            o.w = __shfl_xor_sync(0xffffffffu, r.mine.w, 1);
            bm.ids = half == 0 ? make_int4(r.mine.x, r.mine.z, o.x, o.z)     // rows 0, 2, 4, 6
                               : make_int4(o.y, o.w, r.mine.y, r.mine.w);    // rows 1, 3, 5, 7
            bm.e0 = r.e0;
            bm.e1 = r.e1;
            return bm;
        };
        const Unit kNone = {0, 0, 0, 0, -1, 0, 0, 0};
        auto first_end = [&](const Unit& uu) -> int {
            return (uu.split_id < 0 && uu.wb < uu.we) ? __ldg(rwo + uu.wb + 1) : INT_MAX;
        };
        int32_t* const myctr = uctr ? uctr + 2 * blockIdx.y : nullptr;
        int kst = 0;   // static ordinal
        auto draw = [&]() -> int {   // next unit index (lane 0's value in dynamic mode: shuffle before use)
            if (myctr) return lane == 0 ? atomicAdd(myctr, 1) : 0;
            if (gridDim.x == num_units) return kst++ == 0 ? (int)blockIdx.x : num_units;
            return (int)blockIdx.x + (kst++) * (int)gridDim.x;
        };
        auto bcast = [&](int v) -> int { return myctr ? __shfl_sync(0xffffffffu, v, 0) : v; };
        int q0 = draw();
        int q1 = draw();
        q0 = bcast(q0);
        q1 = bcast(q1);
        Unit u = q0 < num_units ? units[q0] : kNone;
        Unit un = q1 < num_units ? units[q1] : kNone;
        int end0, end0n = INT_MAX;
        Raw rnext;
        if (ufirst && q0 < num_units) {
            // first unit of a one-CTA-per-unit launch: its first batch's SparseAtoB ids, TCOffset
            // bounds and first-window end come from the unit's side record (indexed by blockIdx.x),
            // so they load in parallel with the unit record instead of after it
            const int32_t* fr = ufirst + (int64_t)q0 * kFirstRec;
            rnext.mine = __ldg(reinterpret_cast<const int4*>(fr + jl * 8) + half);
            rnext.e0 = rnext.e1 = 0;
            if (lane == 0) {
                rnext.e0 = __ldg(fr + kPadBatch * 8);
                rnext.e1 = __ldg(fr + kPadBatch * 8 + 1);
            }
            end0 = __ldg(fr + kPadBatch * 8 + 2);
        } else {
            end0 = first_end(u);
            rnext = load_raw(u, 0);
        }
        int gi0 = 0, gc0 = 0;
        for (int ord = 0;; ++ord) {
        // publish unit ord to the consumers (index -1 = no more units)
        if (ord >= 2) mbar_wait(&bar_uempty[ord & 1], ((ord >> 1) - 1) & 1);
        if (lane == 0) {
            int* su = s_unit[ord & 1];
            su[0] = u.wb; su[1] = u.we; su[2] = u.bb; su[3] = u.be;
            su[4] = u.split_id; su[5] = u.piece; su[6] = u.npieces; su[7] = u.slot_base;
            su[8] = end0;
            su[9] = q0 < num_units ? q0 : -1;
            mbar_arrive(&bar_ufull[ord & 1]);
        }
        if (q0 >= num_units) break;
        const int q2 = draw();   // reserve the unit after next now; its latency hides behind this unit
        const int nblocks = u.be - u.bb;
        for (int i0 = 0; i0 < nblocks; i0 += kPadBatch) {
            const int c = gc0 + i0 / kPadBatch, aslot = c & 1;
            const BatchMeta cur = finish(rnext);
            rnext = i0 + kPadBatch < nblocks ? load_raw(u, i0 + kPadBatch) : load_raw(un, 0);
            if (i0 == 0) end0n = first_end(un);
            const int nj = min(kPadBatch, nblocks - i0);
            if (c >= 2) mbar_wait(&bar_aempty[aslot], ((c >> 1) - 1) & 1);
            if (lane == 0) {
                const int64_t lo = ((int64_t)cur.e0 * ELT) & ~int64_t(15);
                const int64_t hi = ((int64_t)cur.e1 * ELT + 15) & ~int64_t(15);
                const uint32_t vbytes = (uint32_t)(hi - lo), mbytes = (uint32_t)nj * 16;
                const uint32_t ibytes = NL > 0 ? (uint32_t)nj * 32 : 0u;
                const uint32_t dst = aring + aslot * kPadASlot;
                s_abyte[aslot] = (int)((int64_t)cur.e0 * ELT - lo);
                mbar_arrive_tx(&bar_afull[aslot], vbytes + mbytes + ibytes);
                if (NL > 0)
                    asm volatile(
                        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                            dst + kPadAIdsOff),
                        "l"(atob + (int64_t)(u.bb + i0) * 8), "r"(ibytes), "r"(smem_u32(&bar_afull[aslot]))
                        : "memory");
                asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                             ::"r"(dst), "l"(reinterpret_cast<const uint8_t*>(avals) + lo), "r"(vbytes),
                             "r"(smem_u32(&bar_afull[aslot])) : "memory");
                asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                             ::"r"(dst + kPadAValBytes), "l"(mask + u.bb + i0), "r"(mbytes),
                             "r"(smem_u32(&bar_afull[aslot])) : "memory");
            }
            for (int j = 0; j < nj; ++j) {
                const int i = gi0 + i0 + j, s = i % R;
                if (i >= R) mbar_wait(&bar_empty[s], ((i / R) - 1) & 1);
                if (tr && i == 0 && lane == 0) tr[3] = gtimer();
                if (lsur > 0 && i % lsur == lsur - 1) {
                    // dual-engine gather: this block's rows go through the LSU path (cp.async 16 B
                    // per lane-chunk, zero-filled for -1 ids and past N) into the same padded stage,
                    // tracked by the stage's mbarrier -- the TMA unit is the per-SM limit otherwise
                    const int r = lane >> 2, srcl = 2 * j + (r & 1);
                    const int ix = __shfl_sync(0xffffffffu, cur.ids.x, srcl), iy = __shfl_sync(0xffffffffu, cur.ids.y, srcl);
                    const int iz = __shfl_sync(0xffffffffu, cur.ids.z, srcl), iw = __shfl_sync(0xffffffffu, cur.ids.w, srcl);
                    const int q = r >> 1;
                    const int id = q == 0 ? ix : q == 1 ? iy : q == 2 ? iz : iw;
                    const char* srow = reinterpret_cast<const char*>(B) + (int64_t)(id < 0 ? 0 : id) * ldb * ELT;
                    const int64_t rowb = N * ELT;
                    for (int sl = 0; sl < nsl; ++sl) {
                        const uint32_t dst = ring + s * STAGE + sl * SLB + (r & 1) * ODD + q * ROWB;
                        const int64_t cb = col0 * ELT + (int64_t)sl * SEG * 128;
#pragma unroll
                        for (int k = 0; k < 2 * SEG; ++k) {
                            const int ch = (lane & 3) + 4 * k;
                            const int64_t off = cb + ch * 16;
                            const int64_t rem = rowb - off;
                            const uint32_t n = id < 0 ? 0u : (rem >= 16 ? 16u : (rem > 0 ? (uint32_t)rem : 0u));
                            asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst + ch * 16),
                                         "l"(n ? srow + off : reinterpret_cast<const char*>(B)), "r"(n) : "memory");
                        }
                    }
                    asm volatile("cp.async.mbarrier.arrive.shared::cta.b64 [%0];" ::"r"(smem_u32(&bar_full[s])) : "memory");
                    __syncwarp();
                    if (lane == 0) mbar_arrive(&bar_full[s]);
                    __syncwarp();
                    continue;
                }
                if (lane == 0) mbar_arrive_tx(&bar_full[s], tx);
                __syncwarp();
                if (jl == j) {
                    for (int sl = 0; sl < nsl; ++sl) {
                        const uint32_t dst = ring + s * STAGE + sl * SLB + half * ODD;
                        asm volatile(
                            "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes"
                            " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(dst),
                            "l"(&bmap), "r"(tcol + sl * tslice), "r"(cur.ids.x), "r"(cur.ids.y), "r"(cur.ids.z),
                            "r"(cur.ids.w), "r"(smem_u32(&bar_full[s]))
                            : "memory");
                    }
                }
                __syncwarp();
            }
        }
        if (nblocks == 0) {
            rnext = load_raw(un, 0);
            end0n = first_end(un);
        }
        gi0 += nblocks;
        gc0 += (nblocks + kPadBatch - 1) / kPadBatch;
        q0 = q1;
        u = un;
        end0 = end0n;
        q1 = bcast(q2);
        un = q1 < num_units ? units[q1] : kNone;
        }
        if (myctr && lane == 0) {   // the last CTA of the column group resets its counter
            __threadfence();
            if (atomicAdd(myctr + 1, 1) == (int)gridDim.x - 1) {
                atomicExch(myctr, 0);
                atomicExch(myctr + 1, 0);
            }
        }
        if (tr && lane == 0) {
            tr[6] = gi0;
            tr[7] = gtimer();
        }
        return;
    }
    if (NL > 0 && warp >= WT) {
        // ================= hybrid register-gather warp (S1 from the A batch, S2 on the LSU path)
        const int g = lane >> 2, t = lane & 3;
        constexpr int VW = Tr::VW;
        const int64_t n0 = col0 + SL * SLICE_COLS + (int64_t)(warp - WT) * CW * COLW1;
        const bool active = n0 < N;
        const int64_t bcol = n0 + (int64_t)VW * g;
        const int64_t base = n0 + 2 * NJ1 * t;
        const int hoff = NJ1;
        const int pos = 8 * (g & 3) + 2 * t;
        const uint32_t below = (1u << pos) - 1u;
        const bool upper = g >= 4;
        const char* bthr = reinterpret_cast<const char*>(B) + bcol * (int64_t)ELT;
        const uint64_t ldb_bytes = (uint64_t)ldb * ELT;
        auto gather = [&](int row, int cw) -> V16 {
            const bool ok = active && row >= 0 && (bcol + cw * COLW1) < N;
            const char* p = ok ? bthr + (uint64_t)(uint32_t)row * ldb_bytes + cw * COLW1 * ELT
                               : reinterpret_cast<const char*>(g_zero_line);
            const uint4 x = __ldg(reinterpret_cast<const uint4*>(p));
            V16 v;
            v.w[0] = x.x; v.w[1] = x.y; v.w[2] = x.z; v.w[3] = x.w;
            return v;
        };
        int gc0 = 0;
        for (int ui = blockIdx.x; ui < num_units; ui += gridDim.x) {
        const Unit u = units[ui];
        const int nblocks = u.be - u.bb;
        const bool split = u.split_id >= 0;
        float acc[NJ][4];
#pragma unroll
        for (int jx = 0; jx < NJ; ++jx) acc[jx][0] = acc[jx][1] = acc[jx][2] = acc[jx][3] = 0.f;
        int cur = u.wb;
        int next_end = INT_MAX;
        if (!split) {
            while (cur < u.we && rwo[cur + 1] <= u.bb) {
                if (active) store_tile<NJ, VEC, QPC, COLW1>(C, ldc, M, N, cur, g, base, hoff, acc, true, rowmap);
                ++cur;
            }
            next_end = cur < u.we ? rwo[cur + 1] : INT_MAX;
        }
        uint32_t vaddr = 0, maddr = 0, iaddr = 0, niaddr = 0;
        V16 b0[CW], b1[CW];
        if (nblocks > 0) {
            mbar_wait(&bar_afull[gc0 & 1], (gc0 >> 1) & 1);
            const uint32_t slot = aring + (gc0 & 1) * kPadASlot;
            vaddr = slot + s_abyte[gc0 & 1];
            maddr = slot + kPadAValBytes;
            iaddr = niaddr = slot + kPadAIdsOff;
            const uint2 id = lds64(iaddr + 8 * t);
#pragma unroll
            for (int cw = 0; cw < CW; ++cw) { b0[cw] = gather((int)id.x, cw); b1[cw] = gather((int)id.y, cw); }
        }
        for (int i = 0; i < nblocks; ++i) {
            const int j = i % kPadBatch, c = gc0 + i / kPadBatch;
            // A fragment of block i (batch c)
            const uint4 m = lds128(maddr + j * 16);
            const uint32_t wl = upper ? m.y : m.x, wh = upper ? m.w : m.z;
            const int c0 = __popc(m.x), c01 = c0 + __popc(m.y);
            const int rl = (upper ? c0 : 0) + __popc(wl & below);
            const int rh = c01 + (upper ? __popc(m.z) : 0) + __popc(wh & below);
            const bool p00 = (wl >> pos) & 1u, p01 = (wl >> (pos + 1)) & 1u;
            const bool p10 = (wh >> pos) & 1u, p11 = (wh >> (pos + 1)) & 1u;
            uint32_t a[FW];
            if constexpr (DT == DTC_TF32) {
                a[0] = to_tf32(__uint_as_float(lds32_pred(vaddr + 4 * rl, p00)));
                a[1] = to_tf32(__uint_as_float(lds32_pred(vaddr + 4 * rh, p10)));
                a[2] = to_tf32(__uint_as_float(lds32_pred(vaddr + 4 * (rl + p00), p01)));
                a[3] = to_tf32(__uint_as_float(lds32_pred(vaddr + 4 * (rh + p10), p11)));
            } else {
                a[0] = lds16_pred(vaddr + 2 * rl, p00) | (lds16_pred(vaddr + 2 * (rl + p00), p01) << 16);
                a[1] = lds16_pred(vaddr + 2 * rh, p10) | (lds16_pred(vaddr + 2 * (rh + p10), p11) << 16);
            }
            vaddr += ELT * (c01 + __popc(m.z) + __popc(m.w));
            // B rows of block i+1 (its ids may live in the next batch)
            V16 n0v[CW], n1v[CW];
            if (i + 1 < nblocks) {
                const int jn = (i + 1) % kPadBatch;
                if (jn == 0) {
                    const int cn = c + 1;
                    mbar_wait(&bar_afull[cn & 1], (cn >> 1) & 1);
                    niaddr = aring + (cn & 1) * kPadASlot + kPadAIdsOff;
                }
                const uint2 id = lds64(niaddr + jn * 32 + 8 * t);
#pragma unroll
                for (int cw = 0; cw < CW; ++cw) { n0v[cw] = gather((int)id.x, cw); n1v[cw] = gather((int)id.y, cw); }
            }
            if (active) {
                if constexpr (DT == DTC_TF32) {
                    const uint32_t aa[4] = {a[0], a[1], a[2], a[3]};
#pragma unroll
                    for (int cw = 0; cw < CW; ++cw)
#pragma unroll
                        for (int jj = 0; jj < NJ1; ++jj) mma_tf32(acc[cw * NJ1 + jj], aa, b0[cw].w[jj], b1[cw].w[jj]);
                } else {
                    const uint32_t aa[2] = {a[0], a[1]};
#pragma unroll
                    for (int cw = 0; cw < CW; ++cw)
#pragma unroll
                        for (int jj = 0; jj < NJ1; ++jj) {
                            const uint32_t bb = __byte_perm(b0[cw].w[jj >> 1], b1[cw].w[jj >> 1], (jj & 1) ? 0x7632 : 0x5410);
                            mma_f16(acc[cw * NJ1 + jj], aa, bb);
                        }
                }
            }
#pragma unroll
            for (int cw = 0; cw < CW; ++cw) { b0[cw] = n0v[cw]; b1[cw] = n1v[cw]; }
            if (j == kPadBatch - 1 || i == nblocks - 1) {   // done with batch c (values, masks, ids)
                __syncwarp();
                if (lane == 0) mbar_arrive(&bar_aempty[c & 1]);
                if (i + 1 < nblocks) {
                    const uint32_t slot = aring + ((c + 1) & 1) * kPadASlot;
                    vaddr = slot + s_abyte[(c + 1) & 1];
                    maddr = slot + kPadAValBytes;
                }
            }
            if (u.bb + i + 1 == next_end) {
                if (active) store_tile<NJ, VEC, QPC, COLW1>(C, ldc, M, N, cur, g, base, hoff, acc, false, rowmap);
#pragma unroll
                for (int jj = 0; jj < NJ; ++jj) acc[jj][0] = acc[jj][1] = acc[jj][2] = acc[jj][3] = 0.f;
                ++cur;
                while (cur < u.we && rwo[cur + 1] == rwo[cur]) {
                    if (active) store_tile<NJ, VEC, QPC, COLW1>(C, ldc, M, N, cur, g, base, hoff, acc, true, rowmap);
                    ++cur;
                }
                next_end = cur < u.we ? rwo[cur + 1] : INT_MAX;
            }
        }
        gc0 += (nblocks + kPadBatch - 1) / kPadBatch;
        if (!active) continue;
        if (!split) {
            while (cur < u.we) { store_tile<NJ, VEC, QPC, COLW1>(C, ldc, M, N, cur, g, base, hoff, acc, true, rowmap); ++cur; }
        } else {
            split_fixup<NJ, VEC, QPC, COLW1>(u, acc, ws, npad, counters + blockIdx.y * 8 + warp, (int64_t)gridDim.y * 8,
                                             C, ldc, M, N, g, lane, base, hoff, rowmap);
        }
        }
        return;
    }
    if (warp >= ncons) return;

    // ================= consumers (S1 A fragments, S3 mma, S4/S5) =================
    const int g = lane >> 2, t = lane & 3;
    const int sl = warp / WPS;                           // slice of this warp
    const int64_t n0 = col0 + (int64_t)warp * CW * COLW1;
    const int64_t base = n0 + (DT == DTC_TF32 ? 4 : 8) * t;
    const int hoff = DT == DTC_TF32 ? 16 : 32;
    const int pos = 8 * (g & 3) + 2 * t;
    const uint32_t below = (1u << pos) - 1u;
    const bool upper = g >= 4;
    // smem byte offsets of the thread's even row t / odd row t at chunk c(g) of the warp's first segment
    const int cg = (g >> 1) + 4 * (g & 1);
    const uint32_t roff0 = sl * SLB + t * ROWB + (warp % WPS) * CW * 128 + cg * 16;
    const uint32_t roff1 = roff0 + ODD;

    // Units arrive from the producer (s_unit), record and first-window end already loaded, so a
    // unit boundary costs no dependent global load.
    int gi0 = 0, gc0 = 0;
    for (int ord = 0;; ++ord) {
    mbar_wait(&bar_ufull[ord & 1], (ord >> 1) & 1);
    Unit u;
    int end0, uidx;
    {
        const int* su = s_unit[ord & 1];
        u.wb = su[0]; u.we = su[1]; u.bb = su[2]; u.be = su[3];
        u.split_id = su[4]; u.piece = su[5]; u.npieces = su[6]; u.slot_base = su[7];
        end0 = su[8];
        uidx = su[9];
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&bar_uempty[ord & 1]);
    if (uidx < 0) break;
    const int nblocks = u.be - u.bb;
    const bool split = u.split_id >= 0;
    float acc[NJ][4];
#pragma unroll
    for (int j = 0; j < NJ; ++j) acc[j][0] = acc[j][1] = acc[j][2] = acc[j][3] = 0.f;
    int cur = u.wb;
    int next_end = INT_MAX;
    if (!split) {
        int e = end0;
        while (cur < u.we && e <= u.bb) {   // leading empty windows
            store_tile<NJ, VEC, QPC, COLW1>(C, ldc, M, N, cur, g, base, hoff, acc, true, rowmap);
            ++cur;
            e = cur < u.we ? rwo[cur + 1] : INT_MAX;
        }
        next_end = cur < u.we ? e : INT_MAX;
    }
    uint32_t vaddr = 0, maddr = 0;   // A batch: next block's first value (bytes), mask array
    for (int i = 0; i < nblocks; ++i) {
        const int j = i % kPadBatch, c = gc0 + i / kPadBatch;
        if (j == 0) {
            mbar_wait(&bar_afull[c & 1], (c >> 1) & 1);
            const uint32_t slot = aring + (c & 1) * kPadASlot;
            vaddr = slot + s_abyte[c & 1];
            maddr = slot + kPadAValBytes;
        }
        // S1: A fragment from the occupancy mask and the batch's values (ascending local id, C5)
        const uint4 m = lds128(maddr + j * 16);
        const uint32_t wl = upper ? m.y : m.x, wh = upper ? m.w : m.z;
        const int c0 = __popc(m.x), c01 = c0 + __popc(m.y);
        const int rl = (upper ? c0 : 0) + __popc(wl & below);
        const int rh = c01 + (upper ? __popc(m.z) : 0) + __popc(wh & below);
        const bool p00 = (wl >> pos) & 1u, p01 = (wl >> (pos + 1)) & 1u;
        const bool p10 = (wh >> pos) & 1u, p11 = (wh >> (pos + 1)) & 1u;
        uint32_t a[FW];
        if constexpr (DT == DTC_TF32) {
            a[0] = to_tf32(__uint_as_float(lds32_pred(vaddr + 4 * rl, p00)));
            a[1] = to_tf32(__uint_as_float(lds32_pred(vaddr + 4 * rh, p10)));
            a[2] = to_tf32(__uint_as_float(lds32_pred(vaddr + 4 * (rl + p00), p01)));
            a[3] = to_tf32(__uint_as_float(lds32_pred(vaddr + 4 * (rh + p10), p11)));
        } else {
            a[0] = lds16_pred(vaddr + 2 * rl, p00) | (lds16_pred(vaddr + 2 * (rl + p00), p01) << 16);
            a[1] = lds16_pred(vaddr + 2 * rh, p10) | (lds16_pred(vaddr + 2 * (rh + p10), p11) << 16);
        }
        vaddr += ELT * (c01 + __popc(m.z) + __popc(m.w));
        // S2/S3: B fragments from the padded stage, mma
        const int gi = gi0 + i, s = gi % R;
        mbar_wait(&bar_full[s], (gi / R) & 1);
        if (tr && gi == 0 && threadIdx.x == 0) tr[4] = gtimer();
        const uint32_t st = ring + s * STAGE;
#pragma unroll
        for (int cw = 0; cw < CW; ++cw) {
            const uint4 x0 = lds128(st + roff0 + cw * 128);
            const uint4 x1 = lds128(st + roff1 + cw * 128);
            const uint32_t y0[4] = {x0.x, x0.y, x0.z, x0.w};
            const uint32_t y1[4] = {x1.x, x1.y, x1.z, x1.w};
            if constexpr (DT == DTC_TF32) {
                const uint32_t aa[4] = {a[0], a[1], a[2], a[3]};
#pragma unroll
                for (int jj = 0; jj < NJ1; ++jj) mma_tf32(acc[cw * NJ1 + jj], aa, y0[jj & 3], y1[jj & 3]);
            } else {
                const uint32_t aa[2] = {a[0], a[1]};
#pragma unroll
                for (int jj = 0; jj < NJ1; ++jj) {
                    const uint32_t bb = __byte_perm(y0[(jj >> 1) & 3], y1[(jj >> 1) & 3], (jj & 1) ? 0x7632 : 0x5410);
                    mma_f16(acc[cw * NJ1 + jj], aa, bb);
                }
            }
        }
        __syncwarp();
        if (lane == 0) {
            mbar_arrive(&bar_empty[s]);
            if (j == kPadBatch - 1 || i == nblocks - 1) mbar_arrive(&bar_aempty[c & 1]);
        }

        if (u.bb + i + 1 == next_end) {
            store_tile<NJ, VEC, QPC, COLW1>(C, ldc, M, N, cur, g, base, hoff, acc, false, rowmap);
#pragma unroll
            for (int jj = 0; jj < NJ; ++jj) acc[jj][0] = acc[jj][1] = acc[jj][2] = acc[jj][3] = 0.f;
            ++cur;
            while (cur < u.we && rwo[cur + 1] == rwo[cur]) {
                store_tile<NJ, VEC, QPC, COLW1>(C, ldc, M, N, cur, g, base, hoff, acc, true, rowmap);
                ++cur;
            }
            next_end = cur < u.we ? rwo[cur + 1] : INT_MAX;
        }
    }
    if (!split) {
        while (cur < u.we) { store_tile<NJ, VEC, QPC, COLW1>(C, ldc, M, N, cur, g, base, hoff, acc, true, rowmap); ++cur; }
    } else {
        split_fixup<NJ, VEC, QPC, COLW1>(u, acc, ws, npad, counters + blockIdx.y * 8 + warp, (int64_t)gridDim.y * 8, C,
                                         ldc, M, N, g, lane, base, hoff, rowmap);
    }
    gi0 += nblocks;
    gc0 += (nblocks + kPadBatch - 1) / kPadBatch;
    }
    if (tr && threadIdx.x == 0) tr[5] = gtimer();
}

// ============================================================ host side
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static EncodeTiledFn encode_fn() {
    static EncodeTiledFn fn = nullptr;
    static bool tried = false;
    if (!tried) {
        tried = true;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&fn, cudaEnableDefault, &q) != cudaSuccess ||
            q != cudaDriverEntryPointSuccess)
            fn = nullptr;
        cudaGetLastError();
    }
    return fn;
}

// Tensor map of B (K rows x N cols, row stride ldb) for 128-byte x 1-row gather4 boxes.
static bool make_bmap(CUtensorMap* map, const void* B, int64_t K, int64_t N, int64_t ldb, int dtype) {
    EncodeTiledFn enc = encode_fn();
    if (!enc) return false;
    const int elt = elt_size(dtype);
    cuuint64_t dims[2] = {(cuuint64_t)N, (cuuint64_t)K};
    cuuint64_t strides[1] = {(cuuint64_t)(ldb * elt)};
    cuuint32_t box[2] = {(cuuint32_t)(128 / elt), 1};
    cuuint32_t estr[2] = {1, 1};
    CUresult r = enc(map, dtype == DTC_FP16 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2,
                     const_cast<void*>(B), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS;
}

// Tensor map of B viewed as 4-byte elements (fp16 pairs for FP16): K rows x N*elt/4 columns,
// gather4 boxes of kPadBoxElts x 1, no swizzle (rows land 528 bytes apart, see k_spmm_pad).
// TMA element size of the padded path: 8 bytes whenever a B row is a whole number of 8-byte words
// (half the elements per gather4 op of 4-byte elements), else 4 (DTC_PAD_TE=4 forces 4).
static int pad_te(int64_t N, int dtype, int seg) {
    const char* e = getenv("DTC_PAD_TE");
    if (e && atoi(e) == 4 && seg != 8) return 4;
    return ((N * elt_size(dtype)) % 8 == 0) ? 8 : 4;
}

static bool make_bmap_pad(CUtensorMap* map, const void* B, int64_t K, int64_t N, int64_t ldb, int dtype, int seg,
                          int te) {
    EncodeTiledFn enc = encode_fn();
    if (!enc) return false;
    const int elt = elt_size(dtype);
    if (seg == 8 && te != 8) return false;
    const int row_bytes = seg == 2 ? pad_row_bytes<2>() : seg == 4 ? pad_row_bytes<4>() : pad_row_bytes<8>();
    cuuint64_t dims[2] = {(cuuint64_t)(N * elt / te), (cuuint64_t)K};
    cuuint64_t strides[1] = {(cuuint64_t)(ldb * elt)};
    cuuint32_t box[2] = {(cuuint32_t)(row_bytes / te), 1};
    cuuint32_t estr[2] = {1, 1};
    CUresult r = enc(map, te == 4 ? CU_TENSOR_MAP_DATA_TYPE_UINT32 : CU_TENSOR_MAP_DATA_TYPE_INT64, 2,
                     const_cast<void*>(B), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS;
}

// optional per-CTA timeline of the TMA path (dtc_set_trace; diagnostics, profiles/)
static int64_t* g_trace = nullptr;
static int64_t g_trace_cap = 0;

struct LaunchArgs {
    dtc_format* h;
    const void* B;
    int64_t ldb;
    float* C;
    int64_t ldc, N;
    int gy;
    int64_t npad;
    cudaStream_t s;
    int nws, pass_ws;   // direct path: warp slices of N, slices per L2-resident pass
    int seg;            // TMA padded path: 128-byte segments per slice (2, 4 or 8)
    int nl;             // TMA padded path: register-gather (LSU) warps per CTA (hybrid), 0 = none
    int te;             // TMA padded path: TMA element bytes (4 or 8)
};

template <int DT, int WARPS>
static size_t tma_smem_bytes() {
    constexpr int STAGE = WARPS * 1024;
    constexpr int R = kBRingBytes / STAGE > 16 ? 16 : kBRingBytes / STAGE;
    return 1024 + (size_t)R * STAGE + (size_t)2 * kChunk * 32 * Traits<DT>::FRAG_WORDS * 4 + 2 * kChunk * 8 * 4 +
           (kChunk + 1) * 4;
}

template <int DT, int WARPS, bool VEC>
static cudaError_t launch_tma(const LaunchArgs& a, const CUtensorMap& map) {
    const size_t smem = tma_smem_bytes<DT, WARPS>();
    static bool attr = false;
    if (!attr) {
        cudaFuncSetAttribute(k_spmm_tma<DT, WARPS, VEC>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        attr = true;
    }
    dim3 grid((unsigned)a.h->num_units, (unsigned)a.gy);
    k_spmm_tma<DT, WARPS, VEC><<<grid, (WARPS + 2) * 32, smem, a.s>>>(map, a.h->units, a.h->rwo, a.h->tco, a.h->lid,
                                                                      a.h->atob, a.h->vals, a.C, a.ldc, a.h->M, a.N,
                                                                      a.h->ws, a.h->counters, a.npad, a.h->rowmap);
    return cudaGetLastError();
}

template <int DT, int WARPS, bool VEC, int CW>
static cudaError_t launch_ldg(const LaunchArgs& a) {
    const size_t smem = ldg_smem_bytes<DT, WARPS>();
    static bool attr = false;
    if (!attr) {
        cudaFuncSetAttribute(k_spmm_ldg<DT, WARPS, VEC, CW>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        attr = true;
    }
    dim3 grid((unsigned)a.h->num_units, (unsigned)a.gy);
    k_spmm_ldg<DT, WARPS, VEC, CW><<<grid, WARPS * 32, smem, a.s>>>(a.h->units, a.h->rwo, a.h->tco, a.h->lid, a.h->atob,
                                                                a.h->vals, a.B, a.ldb, a.C, a.ldc, a.h->M, a.N,
                                                                a.h->ws, a.h->counters, a.npad, a.h->rowmap);
    return cudaGetLastError();
}

template <int DT, int WARPS, bool VEC, int CW>
static cudaError_t launch_dir(const LaunchArgs& a) {
    constexpr int PD = dir_depth<DT>();
    const int64_t items = a.h->num_units * (int64_t)a.nws;
    const int64_t nblk = (items + WARPS - 1) / WARPS;
    if (nblk > INT_MAX) return cudaErrorInvalidConfiguration;
    k_spmm_dir<DT, WARPS, VEC, CW, PD><<<(unsigned)nblk, WARPS * 32, 0, a.s>>>(
        a.h->units, a.h->rwo, a.h->tco, reinterpret_cast<const uint4*>(a.h->mask), a.h->atob, a.h->vals, a.B, a.ldb,
        a.C, a.ldc, a.h->M, a.N, a.h->ws, a.h->counters, a.npad, a.h->rowmap, (int)a.h->num_units, a.nws,
        a.pass_ws);
    return cudaGetLastError();
}

// Persistent launch of the padded-row path (DTC_PAD_PERS=1 / dtc_set_pad_persistent): one wave of
// CTAs (resident CTAs per SM x SMs, over the column groups), each walking units blockIdx.x,
// blockIdx.x + gridDim.x, ... with its B ring running across unit boundaries.
#ifndef DTC_PAD_PERS_DEFAULT
#define DTC_PAD_PERS_DEFAULT 0
#endif
static int g_pad_pers = -1;
static bool pad_lpt() {   // DTC_PAD_LPT=0 keeps the build order in persistent launches (experiments)
    const char* e = getenv("DTC_PAD_LPT");
    return !(e && atoi(e) == 0);
}
static bool pad_persistent() {
    if (g_pad_pers < 0) {
        const char* e = getenv("DTC_PAD_PERS");
        g_pad_pers = e ? (atoi(e) > 0 ? 1 : 0) : DTC_PAD_PERS_DEFAULT;
    }
    return g_pad_pers == 1;
}

// Dual-engine gather (DTC_PAD_LSU=k): every k-th TC block of a CTA is gathered by the producer warp
// with cp.async (LSU path) instead of TMA gather4; 0 = TMA only.
#ifndef DTC_PAD_FIRST_DEFAULT
#define DTC_PAD_FIRST_DEFAULT 1
#endif
#ifndef DTC_PAD_LSU_DEFAULT
#define DTC_PAD_LSU_DEFAULT 0
#endif
static int pad_lsu_every() {   // read per launch (experiments flip it between calls)
    const char* e = getenv("DTC_PAD_LSU");
    return e ? std::max(0, atoi(e)) : DTC_PAD_LSU_DEFAULT;
}

static bool pad_first() {   // DTC_PAD_FIRST=0/1 (read per launch; experiments flip it between calls)
    const char* e = getenv("DTC_PAD_FIRST");
    return e ? atoi(e) > 0 : DTC_PAD_FIRST_DEFAULT;
}

__global__ void k_units_first(int64_t nu, const Unit* __restrict__ units, const int32_t* __restrict__ atob,
                              const int32_t* __restrict__ tco, const int32_t* __restrict__ rwo,
                              int32_t* __restrict__ out) {
    for (int64_t q = blockIdx.x; q < nu; q += gridDim.x) {
        const Unit u = units[q];
        const int nb = u.be - u.bb;
        int32_t* o = out + q * kFirstRec;
        for (int t = threadIdx.x; t < kFirstRec; t += blockDim.x) {
            int32_t v = 0;
            if (t < kPadBatch * 8) {
                const int i = t / 8;
                v = i < nb ? atob[(int64_t)(u.bb + i) * 8 + (t % 8)] : -1;
            } else if (t == kPadBatch * 8) {
                v = nb > 0 ? tco[u.bb] : 0;
            } else if (t == kPadBatch * 8 + 1) {
                v = nb > 0 ? tco[u.bb + min(kPadBatch, nb)] : 0;
            } else if (t == kPadBatch * 8 + 2) {
                v = (u.split_id < 0 && u.wb < u.we) ? rwo[u.wb + 1] : INT_MAX;
            }
            o[t] = v;
        }
    }
}

static cudaError_t first_records(dtc_format* h, cudaStream_t s) {
    if (h->ufirst || h->num_units == 0) return cudaSuccess;
    int32_t* d = nullptr;
    if (dalloc(&d, (size_t)h->num_units * kFirstRec, s) != DTC_OK) return cudaErrorMemoryAllocation;
    k_units_first<<<(unsigned)std::min<int64_t>(h->num_units, 65535), 128, 0, s>>>(h->num_units, h->units, h->atob,
                                                                                  h->tco, h->rwo, d);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) { dfree(d, s); return e; }
    h->ufirst = d;
    return cudaSuccess;
}

// Unit order for the persistent launch: largest units first (stable; longest-processing-time
// first), so the last units CTAs draw are the smallest and the launch ends evenly.  Built once per
// handle on the host (units are 32 B each) at the first persistent launch; results do not depend on
// the order.
static cudaError_t lpt_units(dtc_format* h, cudaStream_t s) {
    if (h->units_lpt || h->num_units == 0) return cudaSuccess;
    std::vector<Unit> u((size_t)h->num_units);
    cudaError_t e = cudaMemcpyAsync(u.data(), h->units, u.size() * sizeof(Unit), cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) return e;
    std::stable_sort(u.begin(), u.end(), [](const Unit& x, const Unit& y) { return (x.be - x.bb) > (y.be - y.bb); });
    Unit* d = nullptr;
    if (dalloc(&d, u.size(), s) != DTC_OK) return cudaErrorMemoryAllocation;
    e = cudaMemcpyAsync(d, u.data(), u.size() * sizeof(Unit), cudaMemcpyHostToDevice, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) { dfree(d, s); return e; }
    h->units_lpt = d;
    return cudaSuccess;
}

template <int DT, int SL, int SEG, int NL, bool VEC>
static cudaError_t launch_pad(const LaunchArgs& a, const CUtensorMap& map) {
    const size_t smem = pad_smem_bytes<SL, SEG>();
    constexpr int threads = (SL * SEG / 2 + NL + 1) * 32;
    static int per_sm = 0;
    if (!per_sm) {
        cudaFuncSetAttribute(k_spmm_pad<DT, SL, SEG, NL, VEC>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_spmm_pad<DT, SL, SEG, NL, VEC>, threads, smem) !=
                cudaSuccess || per_sm < 1) {
            cudaGetLastError();
            per_sm = 1;
        }
    }
    int64_t gx = a.h->num_units;
    int32_t* uctr = nullptr;
    if (pad_persistent()) {
        const int64_t slots = (int64_t)per_sm * num_sms();
        gx = std::min<int64_t>(gx, std::max<int64_t>(1, slots / a.gy));
        // dynamic unit counters (one pair per column group, self-resetting); the hybrid LSU warps
        // walk a static stride, so NL > 0 stays static
        if (NL == 0 && gx < a.h->num_units) {
            if (a.h->uctr_len < 2 * a.gy) {
                dfree(a.h->uctr, a.s);
                a.h->uctr_len = 0;
                if (dalloc(&a.h->uctr, (size_t)2 * a.gy, a.s) != DTC_OK) return cudaErrorMemoryAllocation;
                cudaError_t e = cudaMemsetAsync(a.h->uctr, 0, sizeof(int32_t) * 2 * a.gy, a.s);
                if (e != cudaSuccess) return e;
                a.h->uctr_len = 2 * a.gy;
            }
            uctr = a.h->uctr;
            if (pad_lpt()) {
                cudaError_t e = lpt_units(a.h, a.s);
                if (e != cudaSuccess) return e;
            }
        }
    }
    const Unit* units = (uctr && a.h->units_lpt) ? a.h->units_lpt : a.h->units;
    const int32_t* ufirst = nullptr;
    if (NL == 0 && gx == a.h->num_units && pad_first()) {
        cudaError_t e = first_records(a.h, a.s);
        if (e != cudaSuccess) return e;
        ufirst = a.h->ufirst;
    }
    dim3 grid((unsigned)gx, (unsigned)a.gy);
    k_spmm_pad<DT, SL, SEG, NL, VEC><<<grid, (SL * SEG / 2 + NL + 1) * 32, smem, a.s>>>(
        map, units, a.h->rwo, a.h->tco, reinterpret_cast<const uint4*>(a.h->mask), a.h->atob, a.h->vals, a.C,
        a.ldc, a.h->M, a.N, a.h->ws, a.h->counters, a.npad, a.h->rowmap,
        (g_trace && (int64_t)grid.x * grid.y <= g_trace_cap) ? g_trace : nullptr, a.B, a.ldb, (int)a.h->num_units,
        uctr, a.te, pad_lsu_every(), ufirst);
    return cudaGetLastError();
}

template <int DT, bool VEC>
static cudaError_t dispatch(int warps, int path, const LaunchArgs& a, const CUtensorMap& map) {
    if (path == 4) {   // warps = TMA slices per CTA, a.seg = segments per slice, a.nl = LSU warps
        if (a.nl > 0) {   // hybrid TMA + LSU gathers
            if (a.seg == 2) return launch_pad<DT, 1, 2, 1, VEC>(a, map);
            if (a.seg == 4) return a.nl >= 2 ? launch_pad<DT, 1, 4, 2, VEC>(a, map) : launch_pad<DT, 1, 4, 1, VEC>(a, map);
            return launch_pad<DT, 1, 8, 4, VEC>(a, map);
        }
        if (a.seg == 8) return warps >= 2 ? launch_pad<DT, 2, 8, 0, VEC>(a, map) : launch_pad<DT, 1, 8, 0, VEC>(a, map);
        switch (warps) {
            case 1: return launch_pad<DT, 1, 4, 0, VEC>(a, map);
            case 2: return launch_pad<DT, 2, 4, 0, VEC>(a, map);
            default: return launch_pad<DT, 4, 4, 0, VEC>(a, map);
        }
    }
    const bool tma = path == 2;
    if (path == 3) {
        constexpr int CW = ldg_colchunks<DT>();
        switch (warps) {
            case 1: return launch_dir<DT, 1, VEC, CW>(a);
            case 2: return launch_dir<DT, 2, VEC, CW>(a);
            case 4: return launch_dir<DT, 4, VEC, CW>(a);
            default: return launch_dir<DT, 8, VEC, CW>(a);
        }
    }
    if (tma) {
        switch (warps) {
            case 1: return launch_tma<DT, 1, VEC>(a, map);
            case 2: return launch_tma<DT, 2, VEC>(a, map);
            case 4: return launch_tma<DT, 4, VEC>(a, map);
            default: return launch_tma<DT, 8, VEC>(a, map);
        }
    }
    constexpr int CW = ldg_colchunks<DT>();
    switch (warps) {
        case 1: return launch_ldg<DT, 1, VEC, CW>(a);
        case 2: return launch_ldg<DT, 2, VEC, CW>(a);
        case 4: return launch_ldg<DT, 4, VEC, CW>(a);
        default: return launch_ldg<DT, 8, VEC, CW>(a);
    }
}

static int64_t l2_bytes() {
    static int64_t v = -1;
    if (v < 0) {
        int dev = 0, x = 0;
        cudaGetDevice(&dev);
        if (cudaDeviceGetAttribute(&x, cudaDevAttrL2CacheSize, dev) != cudaSuccess || x <= 0) {
            cudaGetLastError();
            x = 126 << 20;
        }
        v = x;
    }
    return v;
}

static int g_force_path = -1;   // 1 = register gather via smem A chunks, 2 = TMA gather4, 3 = direct (DTC_SPMM_PATH=ldg|tma|dir)
#ifndef DTC_DEFAULT_PATH
#define DTC_DEFAULT_PATH 4   // TMA padded-row path (falls back to path 1 where TMA cannot describe B)
#endif
static int env_path() {
    const char* e = getenv("DTC_SPMM_PATH");
    return (e && e[0] == 't') ? 2 : (e && e[0] == 'l') ? 1 : (e && e[0] == 'd') ? 3 : (e && e[0] == 'p') ? 4
                                                                                                 : DTC_DEFAULT_PATH;
}

int spmm_launch(dtc_format* h, const void* B, int64_t N, int64_t ldb, float* C, int64_t ldc, cudaStream_t s) {
    if (!h) { set_error("null handle"); return DTC_ERR_INVALID; }
    if (N < 1 || ldb < N || ldc < N) {
        set_error("bad N/ldb/ldc (%lld/%lld/%lld)", (long long)N, (long long)ldb, (long long)ldc);
        return DTC_ERR_INVALID;
    }
    if (h->M == 0) return DTC_OK;
    if (!C || (!B && h->T > 0)) { set_error("null B or C"); return DTC_ERR_INVALID; }
    if (h->num_units == 0) return DTC_OK;
    if (g_force_path < 0) g_force_path = env_path();
    const int elt = elt_size(h->dtype);
    const int VW = 16 / elt;
    // TMA needs a 16-byte aligned base and row pitch; a ragged N is fine (OOB columns zero-fill)
    CUtensorMap map;
    memset(&map, 0, sizeof(map));
    const bool tma_ok = (h->T > 0) && ((uintptr_t)B % 16 == 0) && ((ldb * elt) % 16 == 0) &&
                        h->K < (int64_t(1) << 31) && N < (int64_t(1) << 31);
    int path = g_force_path == 3 ? 3 : 1;
    if (g_force_path == 2 && tma_ok && make_bmap(&map, B, h->K, N, ldb, h->dtype)) path = 2;
    // TMA padded path: 1 KB slices (8-byte TMA elements) when a B row holds >= 1 KB, else 512 B
    int seg = ((N * elt) >= 1024 && (N * elt) % 8 == 0) ? 8 : 4;
    int nl = 0;
    {
        const char* e = getenv("DTC_PAD_SEG");
        if (e && atoi(e) == 4) seg = 4;
        // hybrid (experiments): DTC_PAD_HYB=1 splits each CTA's columns half TMA, half LSU gathers
        const char* hy = getenv("DTC_PAD_HYB");
        if (hy && atoi(hy) == 1) {
            const int64_t rb = N * elt;
            if (rb >= 2048 && rb % 8 == 0) { seg = 8; nl = 4; }       // 1 KB TMA + 1 KB LSU per CTA
            else if (rb >= 1024) { seg = 4; nl = 2; }                 // 512 B + 512 B
            else { seg = 2; nl = 1; }                                 // 256 B + 256 B
        }
    }
    const int te = pad_te(N, h->dtype, seg);
    if (g_force_path == 4 && tma_ok && (N * elt) % 4 == 0 && make_bmap_pad(&map, B, h->K, N, ldb, h->dtype, seg, te))
        path = 4;
    // columns per warp: the 128B-swizzled TMA path one 128-byte slice per warp, the others two
    const int colw_tma = h->dtype == DTC_FP16 ? Traits<DTC_FP16>::COLW : Traits<DTC_TF32>::COLW;
    const int colw_ldg = h->dtype == DTC_FP16 ? Traits<DTC_FP16>::COLW * ldg_colchunks<DTC_FP16>()
                                               : Traits<DTC_TF32>::COLW * ldg_colchunks<DTC_TF32>();
    const int colw = path == 2 ? colw_tma : colw_ldg;
    const int64_t need = (N + colw - 1) / colw;
    int warps = need >= 8 ? 8 : need >= 4 ? 4 : need >= 2 ? (need > 2 ? 4 : 2) : 1;
    int64_t cta_cols = (int64_t)warps * colw;
    if (path == 4) {
        // warps := slices (of seg x 128 bytes of a B row) per CTA; seg/2 consumer warps per slice,
        // at most 4 consumer warps per CTA by default (DTC_PAD_SL overrides the slice cap)
        const int64_t slice_cols = seg * 128 / elt;
        const int64_t nsl = (N + slice_cols - 1) / slice_cols;
        const char* e = getenv("DTC_PAD_SL");
        const int slmax = (e && atoi(e) > 0) ? atoi(e) : 2;
        warps = nsl >= 4 && slmax >= 4 && seg == 4 ? 4 : (nsl >= 2 && slmax >= 2 ? 2 : 1);
        cta_cols = warps * slice_cols;
        if (nl > 0) {
            warps = 1;
            cta_cols = slice_cols + nl * 256 / elt;
        }
    }
    const int64_t gy64 = (N + cta_cols - 1) / cta_cols;
    if (gy64 > 65535) { set_error("N too large"); return DTC_ERR_UNSUPPORTED; }
    const int gy = (int)gy64;
    const int64_t npad = gy64 * cta_cols;
    if (h->num_split > 0) {
        // per (slot, column group, consumer warp) -- or (slot, warp slice) on the direct path
        const int64_t ncnt = h->num_slots * std::max<int64_t>((int64_t)gy * 8, need);
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
    // float4 C stores need an aligned C; the LDG path additionally needs B vectors
    const bool cvec = ((uintptr_t)C % 16 == 0) && (ldc % 4 == 0) && (N % 4 == 0);
    const bool bvec = ((uintptr_t)B % 16 == 0) && (ldb % VW == 0) && (N % VW == 0);
    const bool use_vec = (path == 2 || path == 4) ? cvec : (cvec && bvec);
    // direct path: a pass covers pass_ws warp slices, sized so K x (pass columns) of B stays
    // within ~3/4 of L2 (DTC_PASS_WS overrides: a large value = one unit-major pass)
    const int nws = (int)need;
    int pass_ws = nws;
    if (path == 3) {
        const char* e = getenv("DTC_PASS_WS");
        const int64_t slice_bytes = std::max<int64_t>(h->K, 1) * colw * elt;
        const int64_t fit = (l2_bytes() * 3 / 4) / slice_bytes;
        pass_ws = (int)std::min<int64_t>(nws, std::max<int64_t>(1, fit));
        if (e && atoi(e) > 0) pass_ws = std::min(nws, atoi(e));
    }
    LaunchArgs a{h, B, ldb, C, ldc, N, gy, npad, s, nws, pass_ws, seg, nl, te};
    cudaError_t e;
    if (h->dtype == DTC_FP16)
        e = use_vec ? dispatch<DTC_FP16, true>(warps, path, a, map) : dispatch<DTC_FP16, false>(warps, path, a, map);
    else
        e = use_vec ? dispatch<DTC_TF32, true>(warps, path, a, map) : dispatch<DTC_TF32, false>(warps, path, a, map);
    if (e != cudaSuccess) return cuda_fail(e, "k_spmm launch", __FILE__, __LINE__);
    return DTC_OK;
}

}  // namespace dtc

using namespace dtc;

extern "C" int dtc_spmm(dtc_handle_t h, const void* B, int64_t N, int64_t ldb, float* C, int64_t ldc, void* stream) {
    return spmm_launch(h, B, N, ldb, C, ldc, (cudaStream_t)stream);
}

extern "C" int dtc_spmm_launches_per_call(void) { return 1; }

extern "C" int dtc_set_trace(void* dev_buf, int64_t capacity_ctas) {
    if (capacity_ctas < 0 || (capacity_ctas > 0 && !dev_buf)) { set_error("bad trace buffer"); return DTC_ERR_INVALID; }
    g_trace = capacity_ctas ? reinterpret_cast<int64_t*>(dev_buf) : nullptr;
    g_trace_cap = capacity_ctas;
    return DTC_OK;
}

extern "C" int dtc_set_pad_persistent(int on) {
    const int prev = pad_persistent() ? 1 : 0;
    g_pad_pers = on > 0 ? 1 : 0;
    return prev;
}

extern "C" int dtc_set_spmm_path(int path) {
    if (path < 0 || path > 4) { set_error("unknown spmm path %d", path); return DTC_ERR_INVALID; }
    const int prev = g_force_path < 0 ? 0 : g_force_path;
    g_force_path = path == 0 ? DTC_DEFAULT_PATH : path;
    return prev;
}

// Column chunks for dtc_spmm_host: C(:, cols) depends only on B(:, cols), so the call is pipelined
// over column chunks -- H2D of chunk j+1 runs while chunk j computes and its C chunk goes back
// (PCIe / C2C are full duplex).  Every output element is the same sum in the same order as one
// dtc_spmm over all N columns (the kernels' per-column arithmetic does not depend on N).
// Pitched copies of narrow row pieces run well below the wide-copy rate, and each chunk's kernel
// re-reads the format (A), so chunks keep >= 512 B of a B row, or >= 256 B when the format is
// smaller than B (the kernels are short next to the copies); at most 4 chunks.  Measured on B200,
// dtc_spmm_host e2e (profiles/r01_host_chunks.txt): c2 2 x 256 B +24%, c4 2 x 256 B +27%, c3 2 x 512 B
// +27%, c5 4 x 512 B +58%; c3h (FP16, format 5x B) 2 x 256 B -12%, so it stays unpipelined.
// DTC_HOST_CHUNKS overrides the count (1 = the unpipelined copy-in, kernel, copy-out sequence).
static int host_chunks(const dtc_format* h, int64_t N, int elt, size_t bytes) {
    const int64_t row = N * elt;
    const double fmt_bytes = (double)h->nnz * (elt + 1) + 36.0 * (double)h->T + 4.0 * (double)h->W;
    const double b_bytes = (double)std::max<int64_t>(h->K, 1) * row;
    const int64_t wmin = fmt_bytes < b_bytes ? 256 : 512;
    int64_t c = std::min<int64_t>(4, row / wmin);
    if (bytes < ((size_t)8 << 20)) c = 1;   // small calls: latency, not bandwidth
    if (const char* e = getenv("DTC_HOST_CHUNKS")) c = atoi(e);
    return (int)std::max<int64_t>(1, std::min<int64_t>({c, 16, (N + 31) / 32}));   // widths: multiples of 32 columns
}

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
        {
            uint8_t* sb = nullptr;
            int rc0 = dalloc(&sb, bbytes, s);
            if (rc0) return rc0;
            h->stage_B = sb;
        }
        h->stage_B_bytes = bbytes;
    }
    if (cbytes > h->stage_C_bytes) {
        dfree(h->stage_C, s);
        h->stage_C_bytes = 0;
        {
            int rc0 = dalloc(&h->stage_C, cbytes / sizeof(float), s);
            if (rc0) return rc0;
        }
        h->stage_C_bytes = cbytes;
    }
    const int nch = host_chunks(h, N, elt, bbytes + cbytes);
    // Zero-copy C: when C_host is pinned and mapped, the kernel stores C straight into host memory
    // (posted PCIe writes spread over the kernel) and the copy-out disappears.  It pays when the
    // kernel is long next to the copies (format larger than B: c3 e2e 12.1 -> 10.1 ms) and costs
    // 1-5% otherwise (c2, c4, c5; profiles/r01_host_zc.txt).  DTC_HOST_ZC=0/1 overrides.
    float* Czc = nullptr;
    {
        const double fmt_bytes = (double)h->nnz * (elt + 1) + 36.0 * (double)h->T + 4.0 * (double)h->W;
        bool zc = fmt_bytes > (double)bbytes && bbytes + cbytes >= ((size_t)8 << 20);
        if (const char* e = getenv("DTC_HOST_ZC")) zc = atoi(e) > 0;
        cudaPointerAttributes at{};
        if (zc && cudaPointerGetAttributes(&at, C_host) == cudaSuccess && at.type == cudaMemoryTypeHost &&
            at.devicePointer)
            Czc = reinterpret_cast<float*>(at.devicePointer);
        cudaGetLastError();
    }
    if (Czc) {
        for (auto& hs : h->hstream)
            if (!hs) DTC_CUDA(cudaStreamCreateWithFlags(&hs, cudaStreamNonBlocking));
        for (auto& e : h->hev)
            if (!e) DTC_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
        cudaStream_t sin = h->hstream[0];
        DTC_CUDA(cudaEventRecord(h->hev[32], s));
        DTC_CUDA(cudaStreamWaitEvent(sin, h->hev[32], 0));
        const int64_t units32 = (N + 31) / 32;
        int64_t c0 = 0;
        uint8_t* sb = reinterpret_cast<uint8_t*>(h->stage_B);
        for (int j = 0; j < nch; ++j) {
            const int64_t u = units32 / nch + (j < units32 % nch ? 1 : 0);
            const int64_t nc = std::min<int64_t>(N - c0, u * 32);
            uint8_t* bj = sb + (size_t)h->K * c0 * elt;
            if (h->K > 0)
                DTC_CUDA(cudaMemcpy2DAsync(bj, nc * elt, reinterpret_cast<const uint8_t*>(B_host) + c0 * elt,
                                           ldb * elt, nc * elt, h->K, cudaMemcpyHostToDevice, sin));
            DTC_CUDA(cudaEventRecord(h->hev[j], sin));
            DTC_CUDA(cudaStreamWaitEvent(s, h->hev[j], 0));
            int rc = spmm_launch(h, bj, nc, nc, Czc + c0, ldc, s);
            if (rc) return rc;
            c0 += nc;
        }
        DTC_CUDA(cudaStreamSynchronize(s));
        return DTC_OK;
    }
    if (nch <= 1) {
        if (h->K > 0)
            DTC_CUDA(cudaMemcpy2DAsync(h->stage_B, N * elt, B_host, ldb * elt, N * elt, h->K, cudaMemcpyHostToDevice, s));
        int rc = spmm_launch(h, h->stage_B, N, N, h->stage_C, N, s);
        if (rc) return rc;
        if (h->M > 0)
            DTC_CUDA(cudaMemcpy2DAsync(C_host, ldc * sizeof(float), h->stage_C, N * sizeof(float), N * sizeof(float),
                                       h->M, cudaMemcpyDeviceToHost, s));
        DTC_CUDA(cudaStreamSynchronize(s));
        return DTC_OK;
    }
    for (auto& hs : h->hstream)
        if (!hs) DTC_CUDA(cudaStreamCreateWithFlags(&hs, cudaStreamNonBlocking));
    for (auto& e : h->hev)
        if (!e) DTC_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
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
    uint8_t* sb = reinterpret_cast<uint8_t*>(h->stage_B);
    for (int j = 0; j < nch; ++j) {
        const int64_t u = units32 / nch + (j < units32 % nch ? 1 : 0);
        const int64_t nc = std::min<int64_t>(N - c0, u * 32);
        uint8_t* bj = sb + (size_t)h->K * c0 * elt;                 // K x nc, ldb = nc
        float* cj = h->stage_C + (size_t)h->M * c0;                   // M x nc, ldc = nc
        if (h->K > 0)
            DTC_CUDA(cudaMemcpy2DAsync(bj, nc * elt, reinterpret_cast<const uint8_t*>(B_host) + c0 * elt, ldb * elt,
                                       nc * elt, h->K, cudaMemcpyHostToDevice, sin));
        DTC_CUDA(cudaEventRecord(evb[j], sin));
        DTC_CUDA(cudaStreamWaitEvent(s, evb[j], 0));
        int rc = spmm_launch(h, bj, nc, nc, cj, nc, s);
        if (rc) return rc;
        DTC_CUDA(cudaEventRecord(evk[j], s));
        DTC_CUDA(cudaStreamWaitEvent(sout, evk[j], 0));
        if (h->M > 0)
            DTC_CUDA(cudaMemcpy2DAsync(C_host + c0, ldc * sizeof(float), cj, nc * sizeof(float), nc * sizeof(float),
                                       h->M, cudaMemcpyDeviceToHost, sout));
        c0 += nc;
    }
    DTC_CUDA(cudaEventRecord(evs, sout));
    DTC_CUDA(cudaStreamWaitEvent(s, evs, 0));
    DTC_CUDA(cudaStreamSynchronize(s));
    return DTC_OK;
}
