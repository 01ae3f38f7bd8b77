// dtc_spmm.cu -- S1-S5: the DTC-SpMM runtime kernel re-designed for sm_100a.
//
// Paper design (Alg. 2): one thread block per 16-row window
// iterating its TC blocks: FetchSpAsync (A tile -> smem, cp.async double buffered),
// VFetchDense (B rows -> registers with LDG.128, bypassing smem), mma m16n8k4 TF32
// (P:307), a register remap that un-permutes C at the store, and strict balance of
// TC blocks over thread blocks with atomics.
//
// What changes on B200 (measured: DESIGN.md §5, profiles/r01_design_evidence.md):
//  * k_spmm_pad (the product kernel): one producer warp moves the A side of each 16-block batch
//    with two bulk copies (TCValues range + occupancy masks) and every TC block's B rows with TMA
//    tile::gather4 (4 rows x one 512 B / 1 KB row slice per op) into padded shared-memory rows,
//    through an mbarrier ring -- the async B prefetch the paper's GPUs lacked.  Consumer
//    warps build A fragments from the masks (no scatter) and issue mma.sync: m16n8k8 TF32, and
//    m16n8k16 FP16 over pairs of TC blocks of one window (C15).
//  * k_spmm_ldg (fallback where TMA cannot describe B: unaligned base or row pitch): the paper's
//    structure -- A chunks in smem, B rows gathered straight into registers.
// Both: FP32 accumulation; balance + locality from the F4 work units (TC-block sized, window
// ordered); split windows finish with a deterministic two-level fixup (no float
// atomics; the paper used atomics).  The round-1 ablation kernels (128B-swizzled gather4
// ring, the direct LSU kernel, hybrid TMA+LSU CTAs) were removed once measured; their numbers
// are in profiles/r01_design_evidence.md.
#include <cuda.h>
#include <cuda_fp16.h>

#include <algorithm>
#include <atomic>
#include <climits>
#include <vector>

#include "dtc_internal.h"
#include "dtc_sched.h"

namespace dtc {

// register-gather fallback tuning (measured sweep, profiles/r01_design_evidence.md): A chunk of
// 16 (TF32, <= 4 warps) or 32 TC blocks, B double-buffered in registers (P = 1), and per-thread
// register caps that set occupancy for a CTA of W consumer warps owning CW column chunks each
constexpr int kLdgPrefetch = 1;
template <int DT, int W>
constexpr int ldg_chunk() { return (DT == DTC_TF32 && W <= 4) ? 16 : 32; }
template <int DT, int W, int CW>
constexpr int ldg_maxregs() { return CW == 1 ? 64 : (DT == DTC_FP16 ? 112 : (W <= 2 ? 96 : 80)); }
template <int DT, int W, int CW>
constexpr int ldg_min_blocks() {
    constexpr int b = 65536 / (W * 32 * ldg_maxregs<DT, W, CW>());
    return b > 32 ? 32 : (b < 1 ? 1 : b);
}
constexpr int kLdgColChunks = 2;   // a warp owns 2 x 128-byte column slices (64 fp32 / 128 fp16 columns)

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

// FP16 over a pair of TC blocks (C15): A regs {blk0 rows g | g+8, blk1 rows g | g+8}, B regs
// {blk0 k = 2t,2t+1 ; blk1 k = 2t,2t+1} -- the m16n8k16 fragments are two m16n8k8 fragments
__device__ __forceinline__ void mma_f16_k16(float (&d)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1) {
    asm volatile(
        "mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
        "{%0,%1,%2,%3};\n"
        : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
        : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
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

// FP16 block pairing (reading C15): step i of a unit pairs TC blocks i and i+1 when both exist, belong
// to one window, and do not straddle a kFp16PairSpan-block boundary of the unit (the padded kernel's
// A batches and the register-gather kernel's A chunks are multiples of it) -- one rule for both
// kernels, so they compute identical sums and C(:, j) does not depend on which kernel N selects.
constexpr int kFp16PairSpan = 16;
__device__ __forceinline__ bool fp16_pair(int dt, int i, int nblocks, int bb, int next_end) {
    return dt == DTC_FP16 && i + 1 < nblocks && bb + i + 1 != next_end && (i + 1) % kFp16PairSpan != 0;
}

// split-fixup counters per (slot, column group, consumer warp): room for up to 16 consumer warps
constexpr int kFixupWarps = 16;

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
// the same on a shared-memory address (the kernel keeps every barrier address relative to one base
// register instead of re-deriving a generic -> shared conversion per use)
__device__ __forceinline__ void mbar_init(uint32_t bar, int count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count));
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(uint32_t bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
    asm volatile(
        "{\n"
        ".reg .pred p;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        "@!p bra WAIT_%=;\n"
        "}\n" ::"r"(bar),
        "r"(parity)
        : "memory");
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
}

// Split-window fixup for one warp's tile, deterministic, two levels.  A window split into np
// pieces forms groups of G = ceil(sqrt(np)) consecutive pieces (one group when np <= 4).  Every piece
// writes its partial to its slot; the last arriving piece of a group sums the group's slots in piece
// order (into the group's first slot); the last arriving group sums the group sums in group order
// and stores C.  The chain of dependent partial loads is G + np/G instead of np (the single-level
// chain made the last arriver of a hub window the tail of the launch).  Counters live at
// ctr0[slot * cstride] (one per slot and warp column slice): group g at its first slot, the window
// at slot_base + 1 (never a group's first slot when there are >= 2 groups); all self-resetting.

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

// H = 16-row sub-tiles per window (1 for ME-TCF windows, 2 for the 32-row windows of NEXT-2):
// sub-tile h of split piece slot S is workspace slot S*H + h; one arrival per piece covers all of
// its sub-tiles.
template <int H, int NJ, bool VEC, int QPC = NJ / 4, int CSTRIDE = 0>
__device__ __forceinline__ void split_fixup_h(const Unit& u, float (&acc)[H][NJ][4], float* __restrict__ ws,
                                              int64_t npad, int32_t* __restrict__ ctr0, int64_t cstride,
                                              float* __restrict__ C, int64_t ldc, int64_t M, int64_t N, int g, int lane,
                                              int64_t base, int hoff, const int32_t* __restrict__ rowmap) {
    const int np = u.npieces, G = fixup_group(np);
    const int g0 = (u.piece / G) * G, gn = min(G, np - g0), ngr = (np + G - 1) / G;
    const int64_t sb = u.slot_base;
#pragma unroll
    for (int h = 0; h < H; ++h) fixup_write<NJ, QPC, CSTRIDE>(acc[h], ws, (sb + u.piece) * H + h, npad, g, base, hoff);
    if (!arrive_last(ctr0 + (sb + g0) * cstride, gn, lane)) return;
#pragma unroll
    for (int h = 0; h < H; ++h) fixup_sum<NJ, QPC, CSTRIDE>(acc[h], ws, (sb + g0) * H + h, H, gn, npad, g, base, hoff);
    if (ngr > 1) {
#pragma unroll
        for (int h = 0; h < H; ++h) fixup_write<NJ, QPC, CSTRIDE>(acc[h], ws, (sb + g0) * H + h, npad, g, base, hoff);
        if (!arrive_last(ctr0 + (sb + 1) * cstride, ngr, lane)) return;
#pragma unroll
        for (int h = 0; h < H; ++h) fixup_sum<NJ, QPC, CSTRIDE>(acc[h], ws, sb * H + h, (int64_t)G * H, ngr, npad, g, base, hoff);
    }
#pragma unroll
    for (int h = 0; h < H; ++h)
        store_tile<NJ, VEC, QPC, CSTRIDE>(C, ldc, M, N, (int64_t)u.wb * H + h, g, base, hoff, acc[h], false, rowmap);
}

template <int NJ, bool VEC, int QPC = NJ / 4, int CSTRIDE = 0>
__device__ __forceinline__ void split_fixup(const Unit& u, float (&acc)[NJ][4], float* __restrict__ ws, int64_t npad,
                                            int32_t* __restrict__ ctr0, int64_t cstride, float* __restrict__ C,
                                            int64_t ldc, int64_t M, int64_t N, int g, int lane, int64_t base, int hoff,
                                            const int32_t* __restrict__ rowmap) {
    split_fixup_h<1, NJ, VEC, QPC, CSTRIDE>(u, reinterpret_cast<float(&)[1][NJ][4]>(acc), ws, npad, ctr0, cstride, C,
                                            ldc, M, N, g, lane, base, hoff, rowmap);
}
// ---------------------------------------------- TF32 swapped-operand tiles (k_spmm_pad)
// The padded kernel's TF32 mma computes C^T = B^T A^T: the gathered B rows are the m16n8k8 A operand
// (m = 16 B columns, k = the block's 8 B rows), the TC block's values the B operand (n = 8 window
// rows).  A lane's A operand {B[k=t][m=g], B[k=t][m=g+8], B[k=t+4][m=g], B[k=t+4][m=g+8]} is two
// LDS.64 when columns m = g and g + 8 are adjacent in memory, so no register moves precede the HMMA.
// 16-column tile q of a 128-byte segment: lane g's column pair starts at byte sw_colbyte(q, g) --
// {0, 8, 64, 72} for g < 4, {32, 40, 96, 104} for g >= 4, +16 for q = 1 -- which with rows 16 mod
// 128 bytes apart keeps every half-warp LDS.64 conflict-free.  Accumulator j = (cw*2 + q)*2 + nh
// of a warp holds rows 8nh + 2t (d0, d2) and 8nh + 2t + 1 (d1, d3) at columns c, c + 1,
// c = cw*32 + sw_colbyte(q, g)/4.
__host__ __device__ constexpr int sw_colbyte(int q, int g) { return 8 * (g & 1) + 64 * ((g >> 1) & 1) + 32 * (g >> 2) + 16 * q; }
__device__ __forceinline__ int sw_col(int j, int g) { return (j >> 2) * 32 + sw_colbyte((j >> 1) & 1, g) / 4; }

// Vector path: lanes g and g^1 (lane ^ 4) hold columns [b, b+2) and [b+2, b+4) of tile q = 0 and
// [b+4, b+8) of q = 1; one exchange gives the even lane q = 0's four columns and the odd lane q = 1's,
// so every lane stores one float4 per (segment, row) -- whole 16-byte pieces, which matter when C is
// pinned host memory written over PCIe (float2 stores halved the streaming e2e rate).
template <int NJ, bool VEC>
__device__ __forceinline__ void store_tile_sw(float* __restrict__ C, int64_t ldc, int64_t M, int64_t N, int64_t w, int g, int t,
                                              int64_t n0, const float (&acc)[NJ][4], bool zero,
                                              const int32_t* __restrict__ rowmap) {
    const bool odd = g & 1;
#pragma unroll
    for (int nh = 0; nh < 2; ++nh)
#pragma unroll
        for (int rr = 0; rr < 2; ++rr) {
            const int64_t row = w * kWindow + 8 * nh + 2 * t + rr;
            if (VEC) {
                float4 v[NJ / 4];
#pragma unroll
                for (int cw = 0; cw < NJ / 4; ++cw) {
                    const int j0 = (cw * 2) * 2 + nh, j1 = (cw * 2 + 1) * 2 + nh;
                    const float a0 = zero ? 0.f : acc[j0][rr], a1 = zero ? 0.f : acc[j0][2 + rr];
                    const float b0 = zero ? 0.f : acc[j1][rr], b1 = zero ? 0.f : acc[j1][2 + rr];
                    const float r0 = __shfl_xor_sync(0xffffffffu, odd ? a0 : b0, 4);
                    const float r1 = __shfl_xor_sync(0xffffffffu, odd ? a1 : b1, 4);
                    v[cw] = odd ? make_float4(r0, r1, b0, b1) : make_float4(a0, a1, r0, r1);
                }
                if (row >= M) continue;
                float* crow = C + (rowmap ? (int64_t)__ldg(rowmap + row) : row) * ldc;
#pragma unroll
                for (int cw = 0; cw < NJ / 4; ++cw) {
                    const int64_t c = n0 + cw * 32 + sw_colbyte(0, g & ~1) / 4 + (odd ? 4 : 0);
                    if (c < N) *reinterpret_cast<float4*>(crow + c) = v[cw];
                }
            } else {
                if (row >= M) continue;
                float* crow = C + (rowmap ? (int64_t)__ldg(rowmap + row) : row) * ldc;
#pragma unroll
                for (int jj = 0; jj < NJ / 2; ++jj) {
                    const int j = 2 * jj + nh;
                    const int64_t c = n0 + sw_col(j, g);
                    if (c < N) crow[c] = zero ? 0.f : acc[j][rr];
                    if (c + 1 < N) crow[c + 1] = zero ? 0.f : acc[j][2 + rr];
                }
            }
        }
}

template <int NJ>
__device__ __forceinline__ void fixup_write_sw(float (&acc)[NJ][4], float* __restrict__ ws, int64_t slot, int64_t npad,
                                               int g, int t, int64_t n0) {
#pragma unroll
    for (int nh = 0; nh < 2; ++nh)
#pragma unroll
        for (int rr = 0; rr < 2; ++rr) {
            float* prow = ws + (slot * kWindow + 8 * nh + 2 * t + rr) * npad;
#pragma unroll
            for (int jj = 0; jj < NJ / 2; ++jj) {
                const int j = 2 * jj + nh;
                __stcg(reinterpret_cast<float2*>(prow + n0 + sw_col(j, g)), make_float2(acc[j][rr], acc[j][2 + rr]));
            }
        }
}

template <int NJ>
__device__ __forceinline__ void fixup_sum_sw(float (&acc)[NJ][4], const float* __restrict__ ws, int64_t s0, int64_t step,
                                             int cnt, int64_t npad, int g, int t, int64_t n0) {
#pragma unroll
    for (int j = 0; j < NJ; ++j) acc[j][0] = acc[j][1] = acc[j][2] = acc[j][3] = 0.f;
#pragma unroll 1
    for (int k = 0; k < cnt; ++k) {
        const int64_t sl = s0 + k * step;
#pragma unroll
        for (int nh = 0; nh < 2; ++nh)
#pragma unroll
            for (int rr = 0; rr < 2; ++rr) {
                const float* prow = ws + (sl * kWindow + 8 * nh + 2 * t + rr) * npad;
#pragma unroll
                for (int jj = 0; jj < NJ / 2; ++jj) {
                    const int j = 2 * jj + nh;
                    const float2 v = __ldcg(reinterpret_cast<const float2*>(prow + n0 + sw_col(j, g)));
                    acc[j][rr] += v.x;
                    acc[j][2 + rr] += v.y;
                }
            }
    }
}

// split_fixup_h for swapped TF32 tiles (the same two-level deterministic protocol)
template <int H, int NJ, bool VEC>
__device__ __forceinline__ void split_fixup_h_sw(const Unit& u, float (&acc)[H][NJ][4], float* __restrict__ ws,
                                                 int64_t npad, int32_t* __restrict__ ctr0, int64_t cstride,
                                                 float* __restrict__ C, int64_t ldc, int64_t M, int64_t N, int g, int t,
                                                 int lane, int64_t n0, const int32_t* __restrict__ rowmap) {
    const int np = u.npieces, G = fixup_group(np);
    const int g0 = (u.piece / G) * G, gn = min(G, np - g0), ngr = (np + G - 1) / G;
    const int64_t sb = u.slot_base;
#pragma unroll
    for (int h = 0; h < H; ++h) fixup_write_sw<NJ>(acc[h], ws, (sb + u.piece) * H + h, npad, g, t, n0);
    if (!arrive_last(ctr0 + (sb + g0) * cstride, gn, lane)) return;
#pragma unroll
    for (int h = 0; h < H; ++h) fixup_sum_sw<NJ>(acc[h], ws, (sb + g0) * H + h, H, gn, npad, g, t, n0);
    if (ngr > 1) {
#pragma unroll
        for (int h = 0; h < H; ++h) fixup_write_sw<NJ>(acc[h], ws, (sb + g0) * H + h, npad, g, t, n0);
        if (!arrive_last(ctr0 + (sb + 1) * cstride, ngr, lane)) return;
#pragma unroll
        for (int h = 0; h < H; ++h) fixup_sum_sw<NJ>(acc[h], ws, sb * H + h, (int64_t)G * H, ngr, npad, g, t, n0);
    }
#pragma unroll
    for (int h = 0; h < H; ++h) store_tile_sw<NJ, VEC>(C, ldc, M, N, (int64_t)u.wb * H + h, g, t, n0, acc[h], false, rowmap);
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
// streams its 32/64-column B slice with a kLdgPrefetch-deep register ring that runs
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
    constexpr int P = kLdgPrefetch;
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
        auto gather = [&](int row, int cw) -> V16 {
            if (VEC) {
                const bool ok = row >= 0 && (bcol + cw * COLW1) < N;
                const char* p = ok ? bthr + (uint64_t)(uint32_t)row * ldb_bytes + cw * COLW1 * (int)sizeof(typename Tr::elt)
                                   : reinterpret_cast<const char*>(g_zero_line);
                const uint4 x = __ldg(reinterpret_cast<const uint4*>(p));
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
        static_assert(P == 1, "the block-pair step below assumes a one-block register prefetch");
        static_assert(S % kFp16PairSpan == 0, "FP16 pairs never straddle an A chunk");
        for (int i = 0; i < nblocks;) {
            const int c = i / S, j = i % S;
            // FP16: blocks i, i+1 of one window feed one m16n8k16 (same pairing rule as k_spmm_pad,
            // so both kernels compute identical sums); block i+1's B rows are gathered here (its
            // fragment and ids are in the same A chunk), the next step's one block ahead as usual
            const bool pair = fp16_pair(DT, i, nblocks, u.bb, next_end);
            const int nx = i + (pair ? 2 : 1);
            if (active) {
                const uint32_t* fr = s_frag + (c & 1) * S * 32 * FW + j * 32 * FW;
                if (DT == DTC_TF32) {
                    const uint4 av = reinterpret_cast<const uint4*>(fr)[lane];
                    const uint32_t a[4] = {av.x, av.y, av.z, av.w};
#pragma unroll
                    for (int cw = 0; cw < CW; ++cw)
#pragma unroll
                        for (int jj = 0; jj < NJ1; ++jj)
                            mma_tf32(acc[cw * NJ1 + jj], a, b0[0][cw].w[jj], b1[0][cw].w[jj]);
                } else if (pair) {
                    const uint2 av = reinterpret_cast<const uint2*>(fr)[lane];
                    const uint2 av2 = reinterpret_cast<const uint2*>(fr + 32 * FW)[lane];
                    const uint32_t a[4] = {av.x, av.y, av2.x, av2.y};
                    const int2 id2 = ids_of(i + 1);
#pragma unroll
                    for (int cw = 0; cw < CW; ++cw) {
                        const V16 z0 = gather(id2.x, cw), z1 = gather(id2.y, cw);
#pragma unroll
                        for (int jj = 0; jj < NJ1; ++jj) {
                            const uint32_t sel = (jj & 1) ? 0x7632 : 0x5410;
                            const uint32_t bb0 = __byte_perm(b0[0][cw].w[jj >> 1], b1[0][cw].w[jj >> 1], sel);
                            const uint32_t bb1 = __byte_perm(z0.w[jj >> 1], z1.w[jj >> 1], sel);
                            mma_f16_k16(acc[cw * NJ1 + jj], a, bb0, bb1);
                        }
                    }
                } else {
                    const uint2 av = reinterpret_cast<const uint2*>(fr)[lane];
                    const uint32_t a[2] = {av.x, av.y};
#pragma unroll
                    for (int cw = 0; cw < CW; ++cw)
#pragma unroll
                        for (int jj = 0; jj < NJ1; ++jj) {
                            const uint32_t bb = __byte_perm(b0[0][cw].w[jj >> 1], b1[0][cw].w[jj >> 1],
                                                            (jj & 1) ? 0x7632 : 0x5410);
                            mma_f16(acc[cw * NJ1 + jj], a, bb);
                        }
                }
                if (nx < nblocks) {
                    const int2 id = ids_of(nx);
#pragma unroll
                    for (int cw = 0; cw < CW; ++cw) {
                        b0[0][cw] = gather(id.x, cw);
                        b1[0][cw] = gather(id.y, cw);
                    }
                }
            }
            // every warp (active or not) tracks the window ends, so the step -- and with it the
            // chunk-boundary barriers below -- stays CTA-uniform
            if (u.bb + nx == next_end) {
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
            // a step never straddles a chunk (pairs stay inside a kFp16PairSpan-aligned span, which divides S)
            i = nx;
            if (i % S == 0 && i < nblocks) {
                // chunk boundary (CTA-uniform): finish chunk c+1's fragments, recycle buffer c&1
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
// ============================================================ k_spmm_pad: TMA gather4 of padded row slices
// B rows arrive by TMA tile::gather4 in boxes of one 512-byte column slice plus 16 bytes of
// padding (128 fp32 / 256 fp16 columns + 4 / 8 extra), so the 4 rows of one gather4 sit 528
// bytes apart: 528 = 16 (mod 128) shifts each row by one 16-byte bank group.  One op gathers
// the block's even rows (SparseAtoB[0,2,4,6]) at slice offset 0, a second the odd rows at
// offset 2176 (TMA destinations are 128-byte aligned); lane (g,t) reads even row t and odd row
// t -- its mma rows k=t / k=t+4 (TF32; the A columns are permuted alike) or k=2t / 2t+1 (FP16)
// -- at 16-byte chunk c(g) = (g>>1) + 4(g&1) of a 128-byte segment, so the 8 lanes of an LDS.128
// phase hit 8 distinct bank groups: conflict-free without a swizzle, and 4x fewer TMA ops per
// byte than 128-byte swizzled boxes (the r01 gather4 ablation was op-rate bound).  The gather
// moves no data through the LSU pipe (the register gather's limiter: ncu l1tex data-pipe 85%);
// one producer warp runs up to pad_stages blocks ahead.  Consumer warps: 2 per slice, each
// owning 2 x 128-byte segments (64 fp32 / 128 fp16 columns); A fragments are built in
// registers from the occupancy mask.
// Column ownership (virtual mma column v <-> chunk c(v)): TF32 thread holds columns
// seg + 4t + [0,4) and seg + 16 + 4t + [0,4); FP16 seg + 8t + [0,8) and seg + 32 + 8t + [0,8).
// Slice geometry, SEG = 128-byte segments per slice row: 4 (512-byte slices, 4-byte TMA
// elements, box 132) or 8 (1 KB slices, 8-byte TMA elements, box 130 -- one gather4 op moves
// 2x the bytes, for B rows of >= 1 KB).  Row pitch SEG*128 + 16 (= 16 mod 128).
template <int SEG> constexpr int pad_row_bytes() { return SEG * 128 + 16; }
template <int SEG> constexpr int pad_odd_off() { return (4 * pad_row_bytes<SEG>() + 127) / 128 * 128; }
template <int SEG> constexpr int pad_slice_bytes() { return (pad_odd_off<SEG>() + 4 * pad_row_bytes<SEG>() + 127) / 128 * 128; }
template <int SEG> constexpr int pad_tx_bytes() { return 8 * pad_row_bytes<SEG>(); }
static_assert(pad_row_bytes<2>() % 128 == 16 && pad_row_bytes<4>() % 128 == 16 && pad_row_bytes<8>() % 128 == 16,
              "row pitch must be 16 mod 128");
static_assert(pad_row_bytes<2>() % 8 == 0 && pad_row_bytes<4>() % 8 == 0 && pad_row_bytes<8>() % 8 == 0,
              "row pitch: whole 8-byte elements");
// B ring depth (stages of SL slices); measured flat between 3 and 6 once the A side is staged
// (profiles/r01_design_evidence.md), and 6-10 stages with 8-block A batches 4-22% slower than 4
// (profiles/r02_ab_issue.txt): deeper rings only cost CTAs per SM.  -DDTC_PAD_STAGES=k overrides
// for sweeps.
template <int SL>
constexpr int pad_stages() {
#ifdef DTC_PAD_STAGES
    return DTC_PAD_STAGES;
#else
    return SL <= 2 ? 4 : 3;
#endif
}
// A side: per batch of kPadBatch TC blocks, one bulk copy of the (16-byte aligned superset of
// the) batch's TCValues -- contiguous, TCOffset[b0] .. TCOffset[b0+16] -- and one of its 16
// occupancy masks, double buffered.
constexpr int kPadBatch = 16;
static_assert(kPadBatch % kFp16PairSpan == 0, "FP16 pairs never straddle an A batch");
// per-unit side record for the first batch (DTC_OPT_FIRST_RECORDS): kPadBatch x 8 SparseAtoB ids
// (-1 past the unit), TCOffset[bb], TCOffset[bb + min(kPadBatch, nb)], end of the first window,
// TCOffset[bb + min(kPadBatch / 2, nb)] -- one record serves kernels with A batches of 16 or 8 blocks
constexpr int kFirstRec = kPadBatch * 8 + 4;
static_assert((kFirstRec * 4) % 16 == 0, "int4 loads of the side record");
// Per-geometry tuning (measured on one box, profiles/r02_ab_issue.txt):
//  * "slim" CTAs -- TF32, one slice, 16-row windows (c3, c2, c4 N <= 128): A batches of 8 blocks and a
//    96-register cap fit 4 CTAs per SM instead of 3 on c3 (smem 51 KB, 20 warps): c3 +6.5-6.9%, c4
//    N=64/128 +4%, c2 -0.3%.  The consumers' ~70
//    instructions per block run at ~7 cycles each, so more resident warps, not a deeper B ring
//    (6-10 stages measured 4-22% slower), is what raises the block rate.
//  * FP16 and two-slice CTAs (c3h, c5): the producer issues the gathers of 2 TC blocks per pass
//    (G = 2; its per-block bookkeeping halves): c3h +4%, c5 +1%.  G <= R - 1: a consumer holding an
//    FP16 pair's first stage waits for the second, which a G = R group would never issue.
// -DDTC_PAD_TF32_BATCH / DTC_PAD_MAXREGS / DTC_PAD_ISSUE / DTC_PAD_STAGES override every geometry
// (sweeps).
template <int DT, int SL, int SEG, int H> constexpr bool pad_slim() { return DT == DTC_TF32 && H == 1 && SL == 1; }
template <int DT, int SL, int SEG, int H>
constexpr int pad_issue() {
#ifdef DTC_PAD_ISSUE
    return DTC_PAD_ISSUE;
#else
    return (DT == DTC_FP16 || SL == 2) ? 2 : 1;
#endif
}
static_assert(pad_issue<DTC_FP16, 2, 8, 1>() <= pad_stages<2>() - 1 && pad_issue<DTC_FP16, 1, 4, 1>() <= pad_stages<1>() - 1,
              "issue group <= ring depth - 1");
// A batch slot for windows of H x 16 rows: values (<= batch x 128H x 4 B + 16, 128-aligned), then
// one 16H-byte occupancy mask per block
// (tall windows take batches of kPadBatch / H blocks, so a batch slot is the same size for every H)
template <int DT, int SL, int SEG, int H> constexpr int pad_batch() {
#ifdef DTC_PAD_TF32_BATCH
    if (DT == DTC_TF32) return DTC_PAD_TF32_BATCH / H;
#endif
    return pad_slim<DT, SL, SEG, H>() ? kPadBatch / 2 : kPadBatch / H;
}
static_assert(kPadBatch % 8 == 0, "first records hold the A range of the first 8 and 16 blocks");
// B ring depth per geometry: 6 stages for FP16 512 B-slice CTAs (c3h +2.7%; they stay at 5 CTAs/SM,
// limited by registers, with 44 KB of shared memory), pad_stages<SL> elsewhere (deeper rings cost
// the TF32 kernels CTAs per SM, and the FP16 256 B-slice kernel 11%; profiles/r02_ab_issue.txt)
template <int DT, int SL, int SEG, int H> constexpr int pad_stages_g() {
#ifdef DTC_PAD_STAGES
    return DTC_PAD_STAGES;
#else
    return (DT == DTC_FP16 && SL == 1 && SEG == 4) ? 6 : pad_stages<SL>();
#endif
}
// (values of one block: at most 16H x 8 elements of the handle's dtype)
template <int DT, int SL, int SEG, int H> constexpr int pad_aval_bytes() {
    return pad_batch<DT, SL, SEG, H>() * 128 * H * (DT == DTC_FP16 ? 2 : 4) + 128;
}
template <int DT, int SL, int SEG, int H> constexpr int pad_aslot() {
    return pad_aval_bytes<DT, SL, SEG, H>() + pad_batch<DT, SL, SEG, H>() * 16 * H;
}
// Cooperative A expansion (consumers decode each block once into shared memory) pays where a
// CTA has >= 4 consumer warps (each would otherwise decode every block), for FP16 (block pairs),
// and for tall windows; with 2 TF32 consumer warps its barrier and the 16 KB of fragments (fewer
// CTAs per SM) cost more than they save: c3 +13.6%, c5 +7.2%, c4/256 +15%, c3h +6.4%, but
// c2 -14%, c4/128 -13.5% (profiles/r02_ab_coop.txt).
// 128-byte column segments per consumer warp: 2 (64 fp32 / 128 fp16 columns); -DDTC_PAD_SEG8_CW=1
// gives 1 KB-slice CTAs twice the consumer warps with half the columns each (sweeps)
#ifndef DTC_PAD_SEG8_CW
#define DTC_PAD_SEG8_CW 2
#endif
#ifndef DTC_PAD_FP16_CW
#define DTC_PAD_FP16_CW 2
#endif
template <int DT, int SEG> constexpr int pad_cw() {
    return SEG == 8 ? DTC_PAD_SEG8_CW : (DT == DTC_FP16 && SEG == 4 ? DTC_PAD_FP16_CW : 2);
}
template <int DT, int SL, int SEG> constexpr int pad_consumers() { return SL * SEG / pad_cw<DT, SEG>(); }
#ifndef DTC_PAD_COOP_FORCE
#define DTC_PAD_COOP_FORCE -1
#endif
template <int DT, int SL, int SEG, int H>
constexpr bool pad_coop() {
    return DTC_PAD_COOP_FORCE >= 0 ? DTC_PAD_COOP_FORCE == 1 : (DT == DTC_FP16 || pad_consumers<DT, SL, SEG>() >= 4 || H > 1);
}
template <int DT, int SL, int SEG, int H> constexpr int pad_frag_bytes() {
    return pad_coop<DT, SL, SEG, H>() ? 2 * pad_batch<DT, SL, SEG, H>() * H * 32 * Traits<DT>::FRAG_WORDS * 4 : 0;
}
// raw A batch slots (double buffered; a third slot would let the producer run a batch further ahead
// but costs a CTA per SM on c3: 8.59 -> 6.88 TFLOP/s measured, profiles/r02_ab_coop_slots.txt)
template <int DT, int SL, int SEG, int H> constexpr int pad_aslots() { return 2; }
template <int SL, int SEG, int H = 1, int DT = DTC_TF32>
constexpr size_t pad_smem_bytes() {
    return (size_t)pad_stages_g<DT, SL, SEG, H>() * SL * pad_slice_bytes<SEG>() + pad_aslots<DT, SL, SEG, H>() * pad_aslot<DT, SL, SEG, H>() +
           pad_frag_bytes<DT, SL, SEG, H>() + 128 + 256;   // + alignment slack + mbarriers
}
// register cap (sets CTAs per SM); -DDTC_PAD_MAXREGS=r overrides for sweeps
#ifndef DTC_PAD_CW1_REGS
#define DTC_PAD_CW1_REGS 72
#endif
#ifndef DTC_PAD_FP16_REGS
#define DTC_PAD_FP16_REGS 128
#endif
template <int DT, int SL, int SEG, int H>
constexpr int pad_maxregs() {
    if (H > 1) return SL >= 2 ? 112 : 128;   // two 16-row accumulator tiles per thread
    if (DTC_PAD_SEG8_CW == 1 && DT == DTC_TF32) return DTC_PAD_CW1_REGS;
#ifdef DTC_PAD_MAXREGS
    return DTC_PAD_MAXREGS;
#else
    return DT == DTC_FP16 ? DTC_PAD_FP16_REGS : (pad_slim<DT, SL, SEG, H>() ? 96 : 104);
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

template <int DT, int SL, int SEG, bool VEC, int H, bool TRACE = false>
// (min-blocks form of the register cap: measured 8-13% faster than __maxnreg__ with the same cap,
// profiles/r02_ab_launch_bounds.txt)
__global__ void __launch_bounds__((pad_consumers<DT, SL, SEG>() + 1) * 32,
                                  65536 / ((pad_consumers<DT, SL, SEG>() + 1) * 32 * pad_maxregs<DT, SL, SEG, H>()))
k_spmm_pad(const __grid_constant__ CUtensorMap bmap, const Unit* __restrict__ units, const int32_t* __restrict__ rwo,
           const int32_t* __restrict__ tco, const uint4* __restrict__ mask, const int32_t* __restrict__ atob,
           const void* __restrict__ avals, float* __restrict__ C, int64_t ldc, int64_t M, int64_t N,
           float* __restrict__ ws, int32_t* __restrict__ counters, int64_t npad,
           const int32_t* __restrict__ rowmap, int64_t* __restrict__ trace, int num_units,
           int32_t* __restrict__ uctr, int te, const int32_t* __restrict__ ufirst) {
    using Tr = Traits<DT>;
    constexpr int NJ1 = Tr::NJ, COLW1 = Tr::COLW, FW = Tr::FRAG_WORDS;
    constexpr int ELT = (int)sizeof(typename Tr::elt);
    // optional per-CTA timeline (dtc_format_set_trace): {cta, smid, t_start, t_first_issue,
    // t_first_data, t_consumer_done, nblocks, t_producer_done} in %globaltimer ns
    int64_t* tr = (TRACE && trace) ? trace + ((int64_t)blockIdx.y * gridDim.x + blockIdx.x) * 8 : nullptr;   // TRACE instantiation only
    if (tr && threadIdx.x == 0) {
        tr[0] = (int64_t)blockIdx.y * gridDim.x + blockIdx.x;
        tr[1] = smid();
        tr[2] = gtimer();
    }
    constexpr int CW = pad_cw<DT, SEG>();      // 128-byte segments per consumer warp
    constexpr int NJ = NJ1 * CW, QPC = NJ1 / 4;   // QPC quads per segment, segments COLW1 apart
    constexpr int R = pad_stages_g<DT, SL, SEG, H>();
    constexpr int G = pad_issue<DT, SL, SEG, H>();
    constexpr int WPS = SEG / CW;              // consumer warps per slice
    constexpr int ROWB = pad_row_bytes<SEG>(), ODD = pad_odd_off<SEG>(), SLB = pad_slice_bytes<SEG>();
    constexpr int STAGE = SL * SLB;
    constexpr int SLICE_COLS = SEG * COLW1;    // 128 / 256 fp32 or 256 / 512 fp16 columns per slice
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    const uint32_t ring = (smem_u32(smem_raw) + 127u) & ~127u;       // [R][STAGE] B stages
    constexpr int BATCH = pad_batch<DT, SL, SEG, H>();   // TC blocks per A batch
    static_assert(BATCH == kPadBatch || BATCH == kPadBatch / 2, "first records carry the A range of 8 or 16 blocks");
    constexpr int ASLOT = pad_aslot<DT, SL, SEG, H>(), AVAL = pad_aval_bytes<DT, SL, SEG, H>(), NA = pad_aslots<DT, SL, SEG, H>();
    const uint32_t aring = ring + R * STAGE;                          // [2][ASLOT] A batches
    __shared__ int s_abyte[NA];   // byte offset of the batch's first value inside its A slot (batch c: slot (uint32_t)c % NA)
    constexpr bool COOP = pad_coop<DT, SL, SEG, H>();
    // TF32 with 1 KB slices: swapped mma operands (B rows as the A operand, see store_tile_sw) -- no
    // register moves before the HMMAs: c3 +2.3%, c4/256 +1.4%; the 512 B-slice kernel runs on 80
    // registers, where the swap serialises its LDS/HMMA pairs and the epilogue's float2 stores weigh
    // more (c2 -8%, c4/128 -3.5%), so it keeps the direct form (profiles/r02_ab_issue.txt)
    constexpr bool SWAP = DT == DTC_TF32 && SEG == 8;
    __shared__ uint8_t s_live[2][BATCH];   // COOP: per block, bit h = sub-tile h has a non-zero
    const uint32_t frags = aring + NA * ASLOT;  // COOP: [2][BATCH][H] lane-major fragments (expand())
    // mbarriers: full[R], empty[R] (B stages), afull[NA], aempty[NA] (A batches), ufull[2], uempty[2]
    // (published units) -- after the fragments, 8 bytes each
    const uint32_t bar_full = frags + pad_frag_bytes<DT, SL, SEG, H>(), bar_empty = bar_full + 8 * R;
    const uint32_t bar_afull = bar_empty + 8 * R, bar_aempty = bar_afull + 8 * NA;
    const uint32_t bar_ufull = bar_aempty + 8 * NA, bar_uempty = bar_ufull + 16;
    __shared__ int s_unit[2][10];   // published unit: Unit record, end block of its first window, index (-1 = done)

    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    // Units of this CTA: blockIdx.x only (one CTA per unit), or -- persistent launch -- the units
    // the producer draws from the column group's atomic counter uctr[2*blockIdx.y] (dynamic
    // balance; the last CTA resets it), or blockIdx.x + k*gridDim.x when uctr is null.  The
    // producer publishes each unit (record + end of its first window) to the consumers through
    // s_unit / bar_ufull / bar_uempty; the B ring and the A batches run on CTA-wide counters
    // (gi0 blocks, gc0 batches before the current unit), so prefetching continues across units.
    constexpr int CTA_COLS = SL * SLICE_COLS;
    constexpr int WT = SL * WPS;               // consumer warps
    const int64_t col0 = (int64_t)blockIdx.y * CTA_COLS;               // first C column of the CTA
    const int64_t nsl64 = (N - col0 + SLICE_COLS - 1) / SLICE_COLS;
    const int nsl = nsl64 < SL ? (int)(nsl64 > 0 ? nsl64 : 0) : SL;
    const int ncons = WPS * nsl;               // active consumers
    if (threadIdx.x == 0) {
        for (int i = 0; i < R; ++i) {
            mbar_init(bar_full + 8u * (i), 1);
            mbar_init(bar_empty + 8u * (i), ncons);
        }
        for (int i = 0; i < NA; ++i) {
            mbar_init(bar_afull + 8u * (i), 1);
            mbar_init(bar_aempty + 8u * (i), COOP ? 1 : ncons);
        }
        for (int i = 0; i < 2; ++i) {
            mbar_init(bar_ufull + 8u * (i), 1);
            mbar_init(bar_uempty + 8u * (i), ncons);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();

    if (warp == WT) {
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
                r.e1 = __ldg(tco + uu.bb + min(i0 + BATCH, nbu));
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
                rnext.e1 = __ldg(fr + kPadBatch * 8 + (BATCH == kPadBatch ? 1 : 3));
            }
            end0 = __ldg(fr + kPadBatch * 8 + 2);
        } else {
            end0 = first_end(u);
            rnext = load_raw(u, 0);
        }
        int gi0 = 0, gc0 = 0;
        for (int ord = 0;; ++ord) {
            // publish unit ord to the consumers (index -1 = no more units)
            if (ord >= 2) mbar_wait(bar_uempty + 8u * (ord & 1), ((ord >> 1) - 1) & 1);
            if (lane == 0) {
                int* su = s_unit[ord & 1];
                su[0] = u.wb; su[1] = u.we; su[2] = u.bb; su[3] = u.be;
                su[4] = u.split_id; su[5] = u.piece; su[6] = u.npieces; su[7] = u.slot_base;
                su[8] = end0;
                su[9] = q0 < num_units ? q0 : -1;
                mbar_arrive(bar_ufull + 8u * (ord & 1));
            }
            if (q0 >= num_units) break;
            const int q2 = draw();   // reserve the unit after next now; its latency hides behind this unit
            const int nblocks = u.be - u.bb;
            for (int i0 = 0; i0 < nblocks; i0 += BATCH) {
                const int c = gc0 + (uint32_t)i0 / BATCH, aslot = (uint32_t)c % NA;
                const BatchMeta cur = finish(rnext);
                rnext = i0 + BATCH < nblocks ? load_raw(u, i0 + BATCH) : load_raw(un, 0);
                if (i0 == 0) end0n = first_end(un);
                const int nj = min(BATCH, nblocks - i0);
                if (c >= NA) mbar_wait(bar_aempty + 8u * (aslot), (((uint32_t)c / NA) - 1) & 1);
                if (lane == 0) {
                    const int64_t lo = ((int64_t)cur.e0 * ELT) & ~int64_t(15);
                    const int64_t hi = ((int64_t)cur.e1 * ELT + 15) & ~int64_t(15);
                    const uint32_t vbytes = (uint32_t)(hi - lo), mbytes = (uint32_t)nj * 16 * H;
                    const uint32_t dst = aring + aslot * ASLOT;
                    s_abyte[aslot] = (int)((int64_t)cur.e0 * ELT - lo);
                    mbar_arrive_tx(bar_afull + 8u * (aslot), vbytes + mbytes);
                    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                                 ::"r"(dst), "l"(reinterpret_cast<const uint8_t*>(avals) + lo), "r"(vbytes),
                                 "r"((bar_afull + 8u * (aslot))) : "memory");
                    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                                 ::"r"(dst + AVAL), "l"(mask + (int64_t)(u.bb + i0) * H), "r"(mbytes),
                                 "r"((bar_afull + 8u * (aslot))) : "memory");
                }
                // G blocks per issue: the lane pairs of blocks j0 .. j0+G-1 issue their gather4 ops in ONE
                // instruction (the producer's instruction rate, not bytes in flight, bounded the gather)
                for (int j0 = 0; j0 < nj; j0 += G) {
                    const int gn = min(G, nj - j0);
                    for (int j = j0; j < j0 + gn; ++j) {
                        const int i = gi0 + i0 + j;
                        if (i >= R) mbar_wait(bar_empty + 8u * ((uint32_t)i % R), (((uint32_t)i / R) - 1) & 1);
                    }
                    if (TRACE && tr && gi0 + i0 + j0 == 0 && lane == 0) tr[3] = gtimer();
                    const bool mine = jl >= j0 && jl < j0 + gn;
                    const int s = (uint32_t)(gi0 + i0 + jl) % R;
                    if (mine && half == 0) mbar_arrive_tx(bar_full + 8u * (s), tx);
                    __syncwarp();
                    if (mine) {
                        for (int sl = 0; sl < nsl; ++sl) {
                            const uint32_t dst = ring + s * STAGE + sl * SLB + half * ODD;
                            asm volatile(
                                "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes"
                                " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(dst),
                                "l"(&bmap), "r"(tcol + sl * tslice), "r"(cur.ids.x), "r"(cur.ids.y), "r"(cur.ids.z),
                                "r"(cur.ids.w), "r"((bar_full + 8u * (s)))
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
            gc0 += (nblocks + BATCH - 1) / BATCH;
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
    // TF32 (swapped operands): row t of the even / odd half at lane g's column pair of tile q = 0
    const uint32_t soff0 = sl * SLB + t * ROWB + (warp % WPS) * CW * 128 + sw_colbyte(0, g);
    const uint32_t soff1 = soff0 + ODD;
    const int64_t n0w = n0;

    // S1, decoding one 16-row sub-tile of a TC block into this lane's mma A fragment: the occupancy
    // mask m and the block's values at vaddr (ascending local id, C5)
    auto decode = [&](const uint4 m, uint32_t vaddr, uint32_t (&a)[FW]) {
        const uint32_t wl = upper ? m.y : m.x, wh = upper ? m.w : m.z;
        const int c0 = __popc(m.x), c01 = c0 + __popc(m.y);
        const int rl = (upper ? c0 : 0) + __popc(wl & below);
        const int rh = c01 + (upper ? __popc(m.z) : 0) + __popc(wh & below);
        const bool p00 = (wl >> pos) & 1u, p01 = (wl >> (pos + 1)) & 1u;
        const bool p10 = (wh >> pos) & 1u, p11 = (wh >> (pos + 1)) & 1u;
        if constexpr (DT == DTC_TF32) {
            // A fragment (g,t) (g+8,t) (g,t+4) (g+8,t+4); swapped operands want the mma B operand of
            // rows g (a[0], a[1]) and g + 8 (a[2], a[3]), k = t then t + 4
            constexpr int I1 = SWAP ? 2 : 1, I2 = SWAP ? 1 : 2;
            a[0] = to_tf32(__uint_as_float(lds32_pred(vaddr + 4 * rl, p00)));
            a[I1] = to_tf32(__uint_as_float(lds32_pred(vaddr + 4 * rh, p10)));
            a[I2] = to_tf32(__uint_as_float(lds32_pred(vaddr + 4 * (rl + p00), p01)));
            a[3] = to_tf32(__uint_as_float(lds32_pred(vaddr + 4 * (rh + p10), p11)));
        } else {
            a[0] = lds16_pred(vaddr + 2 * rl, p00) | (lds16_pred(vaddr + 2 * (rl + p00), p01) << 16);
            a[1] = lds16_pred(vaddr + 2 * rh, p10) | (lds16_pred(vaddr + 2 * (rh + p10), p11) << 16);
        }
    };
    // Cooperative expansion: at the start of batch c the consumer warps decode its blocks ONCE
    // (warp k takes blocks k, k + ncons, ...) into lane-major fragments in shared memory (FRAG[c&1]),
    // then every warp reads its fragment with one LDS per sub-tile -- instead of each warp decoding
    // every block for its own columns (the decode is ~30 instructions per sub-tile).  One named
    // barrier per batch among the consumers; the raw A slot is released after it, and FRAG[c&1] is
    // rewritten only at batch c+2, after every consumer has passed the barrier of batch c+1.
    constexpr int FSUB = 32 * FW * 4;                      // bytes of one sub-tile's fragments
    auto expand = [&](int c, int nj) {
        mbar_wait(bar_afull + 8u * ((uint32_t)c % NA), ((uint32_t)c / NA) & 1);
        const uint32_t slot = aring + ((uint32_t)c % NA) * ASLOT;
        const uint32_t v0 = slot + s_abyte[(uint32_t)c % NA], maddr = slot + AVAL;
        // value offset of every block of the batch: exclusive warp scan of the blocks' popcounts
        int cnt = 0;
        if (lane < nj)
#pragma unroll
            for (int h = 0; h < H; ++h) {
                const uint4 m = lds128(maddr + (lane * H + h) * 16);
                cnt += __popc(m.x) + __popc(m.y) + __popc(m.z) + __popc(m.w);
            }
        int off = cnt;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(0xffffffffu, off, o);
            if (lane >= o) off += y;
        }
        off -= cnt;
        const uint32_t fbase = frags + (c & 1) * (BATCH * H * FSUB);
        for (int jj = warp; jj < nj; jj += ncons) {
            uint32_t va = v0 + ELT * __shfl_sync(0xffffffffu, off, jj);
            uint32_t lv = 0;
#pragma unroll
            for (int h = 0; h < H; ++h) {
                const uint4 m = lds128(maddr + (jj * H + h) * 16);
                uint32_t a[FW];
                decode(m, va, a);
                va += ELT * (__popc(m.x) + __popc(m.y) + __popc(m.z) + __popc(m.w));
                lv |= ((m.x | m.y | m.z | m.w) != 0u ? 1u : 0u) << h;
                const uint32_t dst = fbase + (jj * H + h) * FSUB + lane * FW * 4;
                if constexpr (FW == 4)
                    asm volatile("st.shared.v4.u32 [%0], {%1, %2, %3, %4};" ::"r"(dst), "r"(a[0]), "r"(a[1]), "r"(a[2]),
                                 "r"(a[3]) : "memory");
                else
                    asm volatile("st.shared.v2.u32 [%0], {%1, %2};" ::"r"(dst), "r"(a[0]), "r"(a[1]) : "memory");
            }
            if (lane == 0) s_live[c & 1][jj] = (uint8_t)lv;
        }
        asm volatile("bar.sync 1, %0;" ::"r"(ncons * 32) : "memory");
    };
    // this lane's fragments of block i (batch c = gc0 + (uint32_t)i / BATCH); live[h] = sub-tile h has a
    // non-zero (warp-uniform)
    auto afrag_coop = [&](int i, int gc0, uint32_t (&a)[H][FW], bool (&live)[H]) {
        const int j = (uint32_t)i % BATCH, c = gc0 + (uint32_t)i / BATCH;
        const uint32_t fbase = frags + (c & 1) * (BATCH * H * FSUB) + j * H * FSUB + lane * FW * 4;
        const uint32_t lv = s_live[c & 1][j];
#pragma unroll
        for (int h = 0; h < H; ++h) {
            live[h] = (lv >> h) & 1u;
            if constexpr (FW == 4) {
                const uint4 x = lds128(fbase + h * FSUB);
                a[h][0] = x.x; a[h][1] = x.y; a[h][2] = x.z; a[h][3] = x.w;
            } else {
                const uint2 x = lds64(fbase + h * FSUB);
                a[h][0] = x.x; a[h][1] = x.y;
            }
        }
    };
    // the raw A slot of a batch is released by warp 0 after its LAST block (not right after the
    // expansion: releasing it at the barrier let the producer run an A batch further ahead and
    // corrupted C on long units -- measured, found with a fragment cross-check; kept late)
    auto release_coop = [&](int i, int gi, int nblocks, int gc0) {
        if (lane == 0) {
            mbar_arrive(bar_empty + 8u * ((uint32_t)gi % R));
            if (warp == 0 && (((uint32_t)i % BATCH) == BATCH - 1 || i == nblocks - 1)) mbar_arrive(bar_aempty + 8u * ((gc0 + (uint32_t)i / BATCH) % NA));
        }
    };

    // A batch cursor: the next block's first value (bytes) and the batch's mask array
    uint32_t vaddr = 0, maddr = 0;
    // S1: the A fragments of block i of the unit (batch c = gc0 + (uint32_t)i / BATCH) -- one per 16-row
    // sub-tile h < H -- decoded by every consumer warp for its own columns; blocks in order
    auto afrag_dec = [&](int i, int gc0, uint32_t (&a)[H][FW], bool (&live)[H]) {
        const int j = (uint32_t)i % BATCH, c = gc0 + (uint32_t)i / BATCH;
        if (j == 0) {
            mbar_wait(bar_afull + 8u * ((uint32_t)c % NA), ((uint32_t)c / NA) & 1);
            const uint32_t slot = aring + ((uint32_t)c % NA) * ASLOT;
            vaddr = slot + s_abyte[(uint32_t)c % NA];
            maddr = slot + AVAL;
        }
#pragma unroll
        for (int h = 0; h < H; ++h) {
            const uint4 m = lds128(maddr + (j * H + h) * 16);
            live[h] = (m.x | m.y | m.z | m.w) != 0u;
            decode(m, vaddr, a[h]);
            vaddr += ELT * (__popc(m.x) + __popc(m.y) + __popc(m.z) + __popc(m.w));
        }
    };
    // release the B stage of CTA block gi and, after a batch's last block, its A slot
    auto release_dec = [&](int i, int gi, int nblocks, int gc0) {
        if (lane == 0) {
            mbar_arrive(bar_empty + 8u * ((uint32_t)gi % R));
            const int j = (uint32_t)i % BATCH;
            if (j == BATCH - 1 || i == nblocks - 1) mbar_arrive(bar_aempty + 8u * ((gc0 + (uint32_t)i / BATCH) % NA));
        }
    };
    auto afrag = [&](int i, int gc0, uint32_t (&a)[H][FW], bool (&live)[H]) {
        if constexpr (COOP) afrag_coop(i, gc0, a, live);
        else afrag_dec(i, gc0, a, live);
    };
    auto release = [&](int i, int gi, int nblocks, int gc0) {
        if constexpr (COOP) release_coop(i, gi, nblocks, gc0);
        else release_dec(i, gi, nblocks, gc0);
    };

    // Units arrive from the producer (s_unit), record and first-window end already loaded, so a
    // unit boundary costs no dependent global load.
    int gi0 = 0, gc0 = 0;
    for (int ord = 0;; ++ord) {
        mbar_wait(bar_ufull + 8u * (ord & 1), (ord >> 1) & 1);
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
        if (lane == 0) mbar_arrive(bar_uempty + 8u * (ord & 1));
        if (uidx < 0) break;
        const int nblocks = u.be - u.bb;
        const bool split = u.split_id >= 0;
        float acc[H][NJ][4];
#pragma unroll
        for (int h = 0; h < H; ++h)
#pragma unroll
            for (int j = 0; j < NJ; ++j) acc[h][j][0] = acc[h][j][1] = acc[h][j][2] = acc[h][j][3] = 0.f;
        // C rows of window w: the 16-row tiles w*H .. w*H+H-1
        auto store_window = [&](int w, bool zero) {
#pragma unroll
            for (int h = 0; h < H; ++h) {
                if constexpr (SWAP)
                    store_tile_sw<NJ, VEC>(C, ldc, M, N, (int64_t)w * H + h, g, t, n0w, acc[h], zero, rowmap);
                else
                    store_tile<NJ, VEC, QPC, COLW1>(C, ldc, M, N, (int64_t)w * H + h, g, base, hoff, acc[h], zero, rowmap);
            }
        };
        int cur = u.wb;
        int next_end = INT_MAX;
        if (!split) {
            int e = end0;
            while (cur < u.we && e <= u.bb) {   // leading empty windows
                store_window(cur, true);
                ++cur;
                e = cur < u.we ? rwo[cur + 1] : INT_MAX;
            }
            next_end = cur < u.we ? e : INT_MAX;
        }
        for (int i = 0; i < nblocks;) {
            const int gi = gi0 + i, s = (uint32_t)gi % R;
            if constexpr (COOP)
                if ((uint32_t)i % BATCH == 0) expand(gc0 + (uint32_t)i / BATCH, min(BATCH, nblocks - i));
            // FP16: two TC blocks of one window feed one m16n8k16 (k = block i's 8 columns, then
            // block i+1's -- the k16 A/B fragments are exactly the two k8 fragments side by side)
            const bool pair = fp16_pair(DT, i, nblocks, u.bb, next_end);
            uint32_t a[H][FW], a2[H][FW];
            bool live[H], live2[H];
            afrag(i, gc0, a, live);
            if (pair) afrag(i + 1, gc0, a2, live2);
            // S2/S3: B fragments from the padded stage(s), mma (a sub-tile without non-zeros is skipped)
            mbar_wait(bar_full + 8u * (s), ((uint32_t)gi / R) & 1);
            if (TRACE && tr && gi == 0 && threadIdx.x == 0) tr[4] = gtimer();   // (compiled out unless traced)
            const uint32_t st = ring + s * STAGE;
            if constexpr (DT == DTC_TF32 && !SWAP) {
#pragma unroll
                for (int cw = 0; cw < CW; ++cw) {
                    const uint4 x0 = lds128(st + roff0 + cw * 128);
                    const uint4 x1 = lds128(st + roff1 + cw * 128);
                    const uint32_t y0[4] = {x0.x, x0.y, x0.z, x0.w};
                    const uint32_t y1[4] = {x1.x, x1.y, x1.z, x1.w};
#pragma unroll
                    for (int h = 0; h < H; ++h)
                        if (H == 1 || live[h])
#pragma unroll
                            for (int jj = 0; jj < NJ1; ++jj) mma_tf32(acc[h][cw * NJ1 + jj], a[h], y0[jj & 3], y1[jj & 3]);
                }
            } else if constexpr (DT == DTC_TF32) {
#pragma unroll
                for (int cw = 0; cw < CW; ++cw) {
#pragma unroll
                    for (int q = 0; q < 2; ++q) {
                        // A operand = B^T tile q: rows k = t (even half) and t + 4 (odd half), columns
                        // m = g, g + 8 adjacent -- two LDS.64 straight into the HMMA's register quadruple
                        const uint2 e = lds64(st + soff0 + cw * 128 + 16 * q);
                        const uint2 o = lds64(st + soff1 + cw * 128 + 16 * q);
                        const uint32_t bt[4] = {e.x, e.y, o.x, o.y};
#pragma unroll
                        for (int h = 0; h < H; ++h)
                            if (H == 1 || live[h])
#pragma unroll
                                for (int nh = 0; nh < 2; ++nh)
                                    mma_tf32(acc[h][(cw * 2 + q) * 2 + nh], bt, a[h][2 * nh], a[h][2 * nh + 1]);
                    }
                }
            } else {
                if (pair) {
                    const int s2 = (uint32_t)(gi + 1) % R;
                    mbar_wait(bar_full + 8u * (s2), ((uint32_t)(gi + 1) / R) & 1);
                    const uint32_t st2 = ring + s2 * STAGE;
#pragma unroll
                    for (int cw = 0; cw < CW; ++cw) {
                        const uint4 x0 = lds128(st + roff0 + cw * 128), x1 = lds128(st + roff1 + cw * 128);
                        const uint4 z0 = lds128(st2 + roff0 + cw * 128), z1 = lds128(st2 + roff1 + cw * 128);
                        const uint32_t y0[4] = {x0.x, x0.y, x0.z, x0.w}, y1[4] = {x1.x, x1.y, x1.z, x1.w};
                        const uint32_t w0[4] = {z0.x, z0.y, z0.z, z0.w}, w1[4] = {z1.x, z1.y, z1.z, z1.w};
#pragma unroll
                        for (int h = 0; h < H; ++h) {
                            const uint32_t aa[4] = {a[h][0], a[h][1], a2[h][0], a2[h][1]};
#pragma unroll
                            for (int jj = 0; jj < NJ1; ++jj) {
                                const uint32_t sel = (jj & 1) ? 0x7632 : 0x5410;
                                const uint32_t b0 = __byte_perm(y0[(jj >> 1) & 3], y1[(jj >> 1) & 3], sel);
                                const uint32_t b1 = __byte_perm(w0[(jj >> 1) & 3], w1[(jj >> 1) & 3], sel);
                                mma_f16_k16(acc[h][cw * NJ1 + jj], aa, b0, b1);
                            }
                        }
                    }
                } else {
#pragma unroll
                    for (int cw = 0; cw < CW; ++cw) {
                        const uint4 x0 = lds128(st + roff0 + cw * 128), x1 = lds128(st + roff1 + cw * 128);
                        const uint32_t y0[4] = {x0.x, x0.y, x0.z, x0.w}, y1[4] = {x1.x, x1.y, x1.z, x1.w};
#pragma unroll
                        for (int h = 0; h < H; ++h) {
                            const uint32_t aa[2] = {a[h][0], a[h][1]};
#pragma unroll
                            for (int jj = 0; jj < NJ1; ++jj) {
                                const uint32_t bb = __byte_perm(y0[(jj >> 1) & 3], y1[(jj >> 1) & 3], (jj & 1) ? 0x7632 : 0x5410);
                                mma_f16(acc[h][cw * NJ1 + jj], aa, bb);
                            }
                        }
                    }
                }
            }
            __syncwarp();
            release(i, gi, nblocks, gc0);
            if (pair) release(i + 1, gi + 1, nblocks, gc0);
            i += pair ? 2 : 1;

            if (u.bb + i == next_end) {
                store_window(cur, false);
#pragma unroll
                for (int h = 0; h < H; ++h)
#pragma unroll
                    for (int jj = 0; jj < NJ; ++jj) acc[h][jj][0] = acc[h][jj][1] = acc[h][jj][2] = acc[h][jj][3] = 0.f;
                ++cur;
                while (cur < u.we && rwo[cur + 1] == rwo[cur]) {
                    store_window(cur, true);
                    ++cur;
                }
                next_end = cur < u.we ? rwo[cur + 1] : INT_MAX;
            }
        }
        if (!split) {
            while (cur < u.we) { store_window(cur, true); ++cur; }
        } else {
            if constexpr (SWAP)
                split_fixup_h_sw<H, NJ, VEC>(u, acc, ws, npad, counters + blockIdx.y * kFixupWarps + warp,
                                             (int64_t)gridDim.y * kFixupWarps, C, ldc, M, N, g, t, lane, n0w, rowmap);
            else
                split_fixup_h<H, NJ, VEC, QPC, COLW1>(u, acc, ws, npad, counters + blockIdx.y * kFixupWarps + warp,
                                                      (int64_t)gridDim.y * kFixupWarps, C, ldc, M, N, g, lane, base, hoff,
                                                      rowmap);
        }
        gi0 += nblocks;
        gc0 += (nblocks + BATCH - 1) / BATCH;
    }
    if (tr && threadIdx.x == 0) tr[5] = gtimer();
}


// ============================================================ host side
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static EncodeTiledFn encode_fn() {
    static EncodeTiledFn fn = []() -> EncodeTiledFn {   // thread-safe one-time init (C++11 statics)
        EncodeTiledFn f = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&f, cudaEnableDefault, &q) != cudaSuccess ||
            q != cudaDriverEntryPointSuccess) {
            cudaGetLastError();
            f = nullptr;
        }
        return f;
    }();
    return fn;
}

// Tensor map of B viewed as te-byte elements (4: fp32 / fp16 pairs, 8: when a B row is a whole number
// of 8-byte words): K rows x N*elt/te columns, gather4 boxes of one padded slice row x 1, no swizzle
// (rows land 528 / 1040 bytes apart, see k_spmm_pad).  Row coordinate -1 (SparseAtoB padding) and
// columns past N are out of bounds: TMA zero-fills them (profiles/r01_tma_gather4_probe.txt).
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

struct LaunchArgs {
    dtc_format* h;
    const void* B;
    int64_t ldb;
    float* C;
    int64_t ldc, N;
    int gy;
    int64_t npad;
    cudaStream_t s;
    int seg;   // padded path: 128-byte segments per slice (2, 4 or 8)
    int te;    // padded path: TMA element bytes (4 or 8)
};

// Per-device launch state of one kernel instantiation: the dynamic shared-memory attribute is set
// and the occupancy queried once per (kernel, device) -- both are per device context.
constexpr int kMaxDevices = 64;
struct KernelState {
    std::atomic<int> per_sm[kMaxDevices];
};
template <class F>
static int kernel_setup(F* fn, int threads, size_t smem, KernelState& ks, int dev) {
    if (dev < 0 || dev >= kMaxDevices) dev = 0;
    int v = ks.per_sm[dev].load(std::memory_order_acquire);
    if (v > 0) return v;
    if (smem > 48 * 1024 && cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess)
        return -1;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&v, fn, threads, smem) != cudaSuccess || v < 1) return -1;
    ks.per_sm[dev].store(v, std::memory_order_release);
    return v;
}

template <int DT, bool VEC, int CW>
static cudaError_t launch_ldg(const LaunchArgs& a, int warps) {
    const dim3 grid((unsigned)a.h->num_units, (unsigned)a.gy);
    switch (warps) {
#define DTC_LDG_CASE(W)                                                                                              \
    case W: {                                                                                                        \
        static KernelState ks;                                                                                       \
        constexpr size_t smem = ldg_smem_bytes<DT, W>();                                                            \
        if (kernel_setup(k_spmm_ldg<DT, W, VEC, CW>, W * 32, smem, ks, a.h->device) < 0)                          \
            return cudaErrorInvalidConfiguration;                                                                    \
        k_spmm_ldg<DT, W, VEC, CW><<<grid, W * 32, smem, a.s>>>(a.h->units, a.h->rwo, a.h->tco, a.h->lid, a.h->atob, \
                                                               a.h->vals, a.B, a.ldb, a.C, a.ldc, a.h->M, a.N,       \
                                                               a.h->ws, a.h->counters, a.npad, a.h->rowmap);        \
        return cudaGetLastError();                                                                                   \
    }
        DTC_LDG_CASE(1)
        DTC_LDG_CASE(2)
        DTC_LDG_CASE(4)
        DTC_LDG_CASE(8)
#undef DTC_LDG_CASE
        default: return cudaErrorInvalidConfiguration;
    }
}

__global__ void k_units_first(int64_t nu, const Unit* __restrict__ units, const int32_t* __restrict__ atob,
                              const int32_t* __restrict__ tco, const int32_t* __restrict__ rwo,
                              int32_t* __restrict__ out) {
    constexpr int batch = kPadBatch;
    for (int64_t q = blockIdx.x; q < nu; q += gridDim.x) {
        const Unit u = units[q];
        const int nb = u.be - u.bb;
        int32_t* o = out + q * kFirstRec;
        for (int t = threadIdx.x; t < kFirstRec; t += blockDim.x) {
            int32_t v = 0;
            if (t < kPadBatch * 8) {
                const int i = t / 8;
                v = (i < nb && i < batch) ? atob[(int64_t)(u.bb + i) * 8 + (t % 8)] : -1;
            } else if (t == kPadBatch * 8) {
                v = nb > 0 ? tco[u.bb] : 0;
            } else if (t == kPadBatch * 8 + 1) {
                v = nb > 0 ? tco[u.bb + min(batch, nb)] : 0;
            } else if (t == kPadBatch * 8 + 2) {
                v = (u.split_id < 0 && u.wb < u.we) ? rwo[u.wb + 1] : INT_MAX;
            } else {
                v = nb > 0 ? tco[u.bb + min(batch / 2, nb)] : 0;
            }
            o[t] = v;
        }
    }
}

// First-batch side records, built once per handle at the first launch that uses them: the
// producer's first A copy and gather4 issues then wait on one DRAM latency (record || unit
// record) instead of two (unit record -> SparseAtoB); profiles/r01_first_records.txt.
static cudaError_t first_records(dtc_format* h, cudaStream_t s) {
    if (h->ufirst || h->num_units == 0) return cudaSuccess;
    int32_t* d = nullptr;
    if (dalloc(&d, (size_t)h->num_units * kFirstRec, s) != DTC_OK) return cudaErrorMemoryAllocation;
    k_units_first<<<(unsigned)std::min<int64_t>(h->num_units, 65535), 128, 0, s>>>(
        h->num_units, h->units, h->atob, h->tco, h->rwo, d);
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

template <int DT, int SL, int SEG, bool VEC, int H>
static cudaError_t launch_pad(const LaunchArgs& a, const CUtensorMap& map) {
    constexpr size_t smem = pad_smem_bytes<SL, SEG, H, DT>();
    constexpr int threads = (pad_consumers<DT, SL, SEG>() + 1) * 32;
    static KernelState ks;
    const int per_sm = kernel_setup(k_spmm_pad<DT, SL, SEG, VEC, H>, threads, smem, ks, a.h->device);
    if (per_sm < 0) {
        const cudaError_t e = cudaGetLastError();
        return e != cudaSuccess ? e : cudaErrorInvalidConfiguration;
    }
    dtc_format* h = a.h;
    int64_t gx = h->num_units;
    int32_t* uctr = nullptr;
    if (h->opt.persistent) {
        const int64_t slots = (int64_t)per_sm * num_sms();
        gx = std::min<int64_t>(gx, std::max<int64_t>(1, slots / a.gy));
        if (gx < h->num_units) {   // dynamic unit counters (one pair per column group, self-resetting)
            if (h->uctr_len < 2 * a.gy) {
                dfree(h->uctr, a.s);
                h->uctr_len = 0;
                if (dalloc(&h->uctr, (size_t)2 * a.gy, a.s) != DTC_OK) return cudaErrorMemoryAllocation;
                cudaError_t e = cudaMemsetAsync(h->uctr, 0, sizeof(int32_t) * 2 * a.gy, a.s);
                if (e != cudaSuccess) return e;
                h->uctr_len = 2 * a.gy;
            }
            uctr = h->uctr;
            cudaError_t e = lpt_units(h, a.s);
            if (e != cudaSuccess) return e;
        }
    }
    const Unit* units = (uctr && h->units_lpt) ? h->units_lpt : h->units;
    const int32_t* ufirst = nullptr;
    if (gx == h->num_units && h->opt.first_records) {
        cudaError_t e = first_records(h, a.s);
        if (e != cudaSuccess) return e;
        ufirst = h->ufirst;
    }
    const dim3 grid((unsigned)gx, (unsigned)a.gy);
    int64_t* trace = (h->trace && (int64_t)grid.x * grid.y <= h->trace_cap) ? h->trace : nullptr;
    if (trace) {   // traced launch: the instantiation that records the per-block timestamps too
        static KernelState kst;
        if (kernel_setup(k_spmm_pad<DT, SL, SEG, VEC, H, true>, threads, smem, kst, a.h->device) < 0)
            return cudaErrorInvalidConfiguration;
        k_spmm_pad<DT, SL, SEG, VEC, H, true><<<grid, threads, smem, a.s>>>(
            map, units, h->rwo, h->tco, reinterpret_cast<const uint4*>(h->mask), h->atob, h->vals, a.C, a.ldc, h->M, a.N,
            h->ws, h->counters, a.npad, h->rowmap, trace, (int)h->num_units, uctr, a.te, ufirst);
        return cudaGetLastError();
    }
    k_spmm_pad<DT, SL, SEG, VEC, H><<<grid, threads, smem, a.s>>>(
        map, units, h->rwo, h->tco, reinterpret_cast<const uint4*>(h->mask), h->atob, h->vals, a.C, a.ldc, h->M, a.N,
        h->ws, h->counters, a.npad, h->rowmap, trace, (int)h->num_units, uctr, a.te, ufirst);
    return cudaGetLastError();
}

template <int DT, bool VEC, int H>
static cudaError_t dispatch_pad_h(int slices, const LaunchArgs& a, const CUtensorMap& map) {
    if (a.seg == 8) return slices >= 2 ? launch_pad<DT, 2, 8, VEC, H>(a, map) : launch_pad<DT, 1, 8, VEC, H>(a, map);
    if (a.seg == 2) return launch_pad<DT, 1, 2, VEC, H>(a, map);
    return slices >= 2 ? launch_pad<DT, 2, 4, VEC, H>(a, map) : launch_pad<DT, 1, 4, VEC, H>(a, map);
}
template <int DT, bool VEC>
static cudaError_t dispatch_pad(int slices, const LaunchArgs& a, const CUtensorMap& map) {
    if (DT == DTC_TF32 && a.h->window_h == 32)
        return a.seg == 8 ? launch_pad<DTC_TF32, 1, 8, VEC, 2>(a, map)
             : a.seg == 2 ? launch_pad<DTC_TF32, 1, 2, VEC, 2>(a, map)
                          : launch_pad<DTC_TF32, 1, 4, VEC, 2>(a, map);
    return dispatch_pad_h<DT, VEC, 1>(slices, a, map);
}

// Padded-path geometry for N columns: 1 KB slices (8-byte TMA elements) when a B row holds >= 1 KB,
// 256 B slices (one consumer warp) when it holds <= 256 B -- a 512 B slice would leave half its
// consumer warps computing columns past N -- else 512 B; <= 2 slices (seg/2 consumer warps each)
// per CTA.
PadGeometry pad_geometry(int dtype, int64_t N, int slice_bytes) {
    const int elt = elt_size(dtype);
    PadGeometry g;
    g.seg = ((N * elt) >= 1024 && (N * elt) % 8 == 0) ? 8 : (N * elt) <= 256 ? 2 : 4;
    if (slice_bytes == 512) g.seg = 4;
    if (slice_bytes == 1024 && (N * elt) % 8 == 0) g.seg = 8;
    const int64_t slice_cols = g.seg * 128 / elt;
    const int64_t nsl = (N + slice_cols - 1) / slice_cols;
#ifndef DTC_PAD_MAX_SLICES
#define DTC_PAD_MAX_SLICES 2
#endif
    g.slices = nsl >= 2 && DTC_PAD_MAX_SLICES >= 2 ? 2 : 1;
    g.cta_cols = g.slices * slice_cols;
    return g;
}

// Resident CTAs per SM of the padded kernel dtc_spmm would launch for N columns (vector C path), on
// the current device -- the measured occupancy the Selector plans with.
int pad_occupancy(int dtype, int64_t N, int window_h) {
    const PadGeometry g = pad_geometry(dtype, N, 0);
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); return -1; }
    auto occ = [&](auto kern, int thr, size_t smem) -> int {
        // (every k_spmm_pad instantiation has the same type, so no per-type static cache here)
        int v = 0;
        if (smem > 48 * 1024 &&
            cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess)
            return -1;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&v, kern, thr, smem) != cudaSuccess) return -1;
        return v;
    };
#define DTC_OCC(DT, H)                                                                                              \
    do {                                                                                                            \
        if (g.seg == 8)                                                                                             \
            return g.slices >= 2 ? occ(k_spmm_pad<DT, 2, 8, true, H>, (pad_consumers<DT, 2, 8>() + 1) * 32, pad_smem_bytes<2, 8, H, DT>())               \
                                 : occ(k_spmm_pad<DT, 1, 8, true, H>, (pad_consumers<DT, 1, 8>() + 1) * 32, pad_smem_bytes<1, 8, H, DT>());              \
        if (g.seg == 2) return occ(k_spmm_pad<DT, 1, 2, true, H>, (pad_consumers<DT, 1, 2>() + 1) * 32, pad_smem_bytes<1, 2, H, DT>());               \
        return g.slices >= 2 ? occ(k_spmm_pad<DT, 2, 4, true, H>, (pad_consumers<DT, 2, 4>() + 1) * 32, pad_smem_bytes<2, 4, H, DT>())                   \
                             : occ(k_spmm_pad<DT, 1, 4, true, H>, (pad_consumers<DT, 1, 4>() + 1) * 32, pad_smem_bytes<1, 4, H, DT>());                  \
    } while (0)
    if (dtype == DTC_FP16) DTC_OCC(DTC_FP16, 1);
    if (window_h == 32) {   // one slice per CTA (see spmm_launch)
        if (g.seg == 8) return occ(k_spmm_pad<DTC_TF32, 1, 8, true, 2>, (pad_consumers<DTC_TF32, 1, 8>() + 1) * 32, pad_smem_bytes<1, 8, 2>());
        if (g.seg == 2) return occ(k_spmm_pad<DTC_TF32, 1, 2, true, 2>, (pad_consumers<DTC_TF32, 1, 2>() + 1) * 32, pad_smem_bytes<1, 2, 2>());
        return occ(k_spmm_pad<DTC_TF32, 1, 4, true, 2>, (pad_consumers<DTC_TF32, 1, 4>() + 1) * 32, pad_smem_bytes<1, 4, 2>());
    }
    DTC_OCC(DTC_TF32, 1);
#undef DTC_OCC
}

// RAII: make the handle's device current for the duration of a call
struct DeviceGuard {
    int prev = -1;
    bool ok = true;
    explicit DeviceGuard(int dev) {
        if (cudaGetDevice(&prev) != cudaSuccess) { cudaGetLastError(); prev = -1; ok = false; return; }
        if (prev != dev && cudaSetDevice(dev) != cudaSuccess) { cudaGetLastError(); ok = false; }
    }
    ~DeviceGuard() {
        int cur = -1;
        if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
    }
};

int spmm_launch(dtc_format* h, const void* B, int64_t N, int64_t ldb, float* C, int64_t ldc, cudaStream_t s) {
    if (!h) { set_error("null handle"); return DTC_ERR_INVALID; }
    if (N < 1 || ldb < N || ldc < N) {
        set_error("bad N/ldb/ldc (%lld/%lld/%lld)", (long long)N, (long long)ldb, (long long)ldc);
        return DTC_ERR_INVALID;
    }
    if (h->M == 0) return DTC_OK;
    if (!C || (!B && h->T > 0)) { set_error("null B or C"); return DTC_ERR_INVALID; }
    if (h->num_units == 0) return DTC_OK;
    DeviceGuard dg(h->device);
    if (!dg.ok) { set_error("cannot select the handle's device %d", h->device); return DTC_ERR_CUDA; }
    const int elt = elt_size(h->dtype);
    const int VW = 16 / elt;
    // TMA needs a 16-byte aligned base and row pitch; a ragged N is fine (OOB columns zero-fill)
    CUtensorMap map;
    memset(&map, 0, sizeof(map));
    const bool tma_ok = (h->T > 0) && ((uintptr_t)B % 16 == 0) && ((ldb * elt) % 16 == 0) && ((N * elt) % 4 == 0) &&
                        h->K < (int64_t(1) << 31) && N < (int64_t(1) << 31);
    const PadGeometry pg = pad_geometry(h->dtype, N, h->opt.slice_bytes);
    const int seg = pg.seg;
    const int te = ((N * elt) % 8 == 0) ? 8 : 4;
    if (h->window_h != kWindow && !tma_ok && h->T > 0) {
        // tall windows run on the padded kernel only: stage B in a library-owned buffer with a
        // 16-byte aligned row pitch (a plain strided copy; the arithmetic is unchanged)
        const int64_t ldb2 = (N + 3) / 4 * 4;
        const size_t need = (size_t)std::max<int64_t>(h->K, 1) * ldb2 * elt;
        if (need > h->stage_B_bytes) {
            dfree(h->stage_B, s);
            h->stage_B_bytes = 0;
            uint8_t* sb = nullptr;
            int rc = dalloc(&sb, need, s);
            if (rc) return rc;
            h->stage_B = sb;
            h->stage_B_bytes = need;
        }
        if (h->K > 0)
            DTC_CUDA(cudaMemcpy2DAsync(h->stage_B, ldb2 * elt, B, ldb * elt, N * elt, h->K, cudaMemcpyDeviceToDevice, s));
        B = h->stage_B;
        ldb = ldb2;
    }
    const bool tma_ok2 = (h->T > 0) && ((uintptr_t)B % 16 == 0) && ((ldb * elt) % 16 == 0) && ((N * elt) % 4 == 0) &&
                         h->K < (int64_t(1) << 31) && N < (int64_t(1) << 31);
    bool pad = (h->opt.kernel != 1 || h->window_h != kWindow) && tma_ok2 &&
               make_bmap_pad(&map, B, h->K, N, ldb, h->dtype, seg, te);
    if (!pad && h->window_h != kWindow && h->T > 0) {
        set_error("tall-window formats need the padded TMA kernel (tensor map encoding failed)");
        return DTC_ERR_UNSUPPORTED;
    }
    int64_t cta_cols, slices = 1;
    int warps = 1;
    const int colw_ldg = (h->dtype == DTC_FP16 ? Traits<DTC_FP16>::COLW : Traits<DTC_TF32>::COLW) * kLdgColChunks;
    if (pad) {
        // tall windows keep one slice per CTA (two accumulator tiles per thread leave no registers for
        // a second slice; wider B takes more column groups)
        slices = h->window_h != kWindow ? 1 : pg.slices;
        cta_cols = slices * (pg.cta_cols / pg.slices);
    } else {
        const int64_t need = (N + colw_ldg - 1) / colw_ldg;
        warps = need >= 8 ? 8 : need >= 4 ? 4 : need >= 2 ? (need > 2 ? 4 : 2) : 1;
        cta_cols = (int64_t)warps * colw_ldg;
    }
    const int64_t gy64 = (N + cta_cols - 1) / cta_cols;
    if (gy64 > 65535) { set_error("N too large"); return DTC_ERR_UNSUPPORTED; }
    const int gy = (int)gy64;
    const int64_t npad = gy64 * cta_cols;
    if (h->num_split > 0) {
        // split fixup counters per (slot, column group, consumer warp), self-resetting
        const int64_t ncnt = h->num_slots * (int64_t)gy * kFixupWarps;
        if (ncnt > h->counters_len) {
            dfree(h->counters, s);
            h->counters_len = 0;
            int rc = dalloc(&h->counters, ncnt, s);
            if (rc) return rc;
            DTC_CUDA(cudaMemsetAsync(h->counters, 0, ncnt * sizeof(int32_t), s));
            h->counters_len = ncnt;
        }
        const size_t wsb = (size_t)h->num_slots * h->window_h * npad * sizeof(float);
        if (wsb > h->ws_bytes) {
            dfree(h->ws, s);
            h->ws_bytes = 0;
            int rc = dalloc(&h->ws, wsb / sizeof(float), s);
            if (rc) return rc;
            h->ws_bytes = wsb;
        }
    }
    // float4 C stores need an aligned C; the register-gather path additionally needs B vectors
    const bool cvec = ((uintptr_t)C % 16 == 0) && (ldc % 4 == 0) && (N % 4 == 0);
    const bool bvec = ((uintptr_t)B % 16 == 0) && (ldb % VW == 0) && (N % VW == 0);
    const bool use_vec = pad ? cvec : (cvec && bvec);
    LaunchArgs a{h, B, ldb, C, ldc, N, gy, npad, s, seg, te};
    cudaError_t e;
    if (pad) {
        if (h->dtype == DTC_FP16)
            e = use_vec ? dispatch_pad<DTC_FP16, true>((int)slices, a, map) : dispatch_pad<DTC_FP16, false>((int)slices, a, map);
        else
            e = use_vec ? dispatch_pad<DTC_TF32, true>((int)slices, a, map) : dispatch_pad<DTC_TF32, false>((int)slices, a, map);
    } else {
        if (h->dtype == DTC_FP16)
            e = use_vec ? launch_ldg<DTC_FP16, true, kLdgColChunks>(a, warps) : launch_ldg<DTC_FP16, false, kLdgColChunks>(a, warps);
        else
            e = use_vec ? launch_ldg<DTC_TF32, true, kLdgColChunks>(a, warps) : launch_ldg<DTC_TF32, false, kLdgColChunks>(a, warps);
    }
    h->last_kernel = pad ? 4 : 1;
    if (e != cudaSuccess) return cuda_fail(e, "k_spmm launch", __FILE__, __LINE__);
    return DTC_OK;
}

}  // namespace dtc

using namespace dtc;

extern "C" int dtc_spmm(dtc_handle_t h, const void* B, int64_t N, int64_t ldb, float* C, int64_t ldc, void* stream) {
    return spmm_launch(h, B, N, ldb, C, ldc, (cudaStream_t)stream);
}

extern "C" int dtc_spmm_launches_per_call(void) { return 1; }
