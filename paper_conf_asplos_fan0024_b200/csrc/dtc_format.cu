// dtc_format.cu -- F0-F4: CSR -> ME-TCF condensation and the work-unit schedule,
// all on the GPU ("Modules ... accelerated by highly parallel CUDA
// kernels", :457 "we develop GPU kernels to accelerate this process").
//
// ME-TCF (§4.2): RowWindowOffset[W+1], TCOffset[T+1],
// TCLocalId[nnz] (uint8), SparseAtoB[8T]; plus TCValues[nnz] (C7).
// Canonical form (C3-C6): a window's condensed columns are its unique
// original columns in ascending order; local id = row_in_window*8 + col_in_block;
// the nnz of a block are stored by ascending local id; the last block of a
// window is padded with -1.
//
// Pipeline:
//   F0  k_validate        warp per row: rowptr shape, column range/order/dupes
//   F1  k_dedup_sort      CTA per window with <= 2048 nnz: smem bitonic sort + unique
//       k_dedup_bitmap    CTA per larger window: chunked smem bitmap over its column span
//                         -> u_w, the window's ascending unique list, rank of every nnz
//   F2  scan ceil(u_w/8)  -> RowWindowOffset, T                  (host sync #1)
//   F3  k_fill_window: CTA per window -- SparseAtoB, 128-bit occupancy mask per TC block
//       (smem atomics), TCOffset by a CTA scan, position = TCOffset + popcount of lower ids
//   F4  k_units_count + scans + k_units_fill/fix (host sync #2: unit count)
#include <algorithm>
#include <climits>
#include <cstring>
#include <chrono>
#include <new>
#include <vector>

#include <cub/device/device_radix_sort.cuh>

#include "dtc_device.cuh"
#include "dtc_internal.h"
#include "dtc_sched.h"

namespace dtc {

constexpr int kSortMax = 2048;         // windows up to this many nnz take the smem sort path
constexpr int kSortThreads = 256;
constexpr int kBmThreads = 256;
constexpr int kBmWords = 8192;          // 2^18 columns per bitmap chunk
constexpr int kBmBits = kBmWords * 32;

enum : int { F_INVALID = 1, F_UNSORTED = 2, F_DUPLICATE = 4, F_RANGE = 8 };

__device__ __forceinline__ int64_t clamp64(int64_t v, int64_t lo, int64_t hi) {
    return v < lo ? lo : (v > hi ? hi : v);
}

// Window w's nnz segment [s0, s1) (clamped so malformed input cannot fault); windows of WH rows
// (16 = the paper's BLOCK_HEIGHT; 32 = the tall windows of NEXT-2).
template <int WH>
__device__ __forceinline__ void window_segment(const int32_t* rowptr, int64_t M, int64_t nnz, int64_t w,
                                               int64_t* s0, int64_t* s1) {
    int64_t r0 = w * WH, r1 = min(r0 + WH, M);
    int64_t a = clamp64(rowptr[r0], 0, nnz), b = clamp64(rowptr[r1], 0, nnz);
    *s0 = a;
    *s1 = b < a ? a : b;
}

// ---------------------------------------------------------------- F0
__global__ void k_validate(int64_t M, int64_t K, int64_t nnz, const int32_t* __restrict__ rowptr,
                           const int32_t* __restrict__ colidx, int* __restrict__ flags) {
    const int lane = threadIdx.x & 31;
    int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    int f = 0;
    for (int64_t r = warp; r < M; r += nwarps) {
        int64_t lo = rowptr[r], hi = rowptr[r + 1];
        if ((r == 0 && lo != 0) || (r == M - 1 && hi != nnz) || lo < 0 || hi > nnz || lo > hi) {
            f |= F_INVALID;
            continue;
        }
        for (int64_t p = lo + lane; p < hi; p += 32) {
            int c = colidx[p];
            if (c < 0 || c >= K) f |= F_RANGE;
            if (p > lo) {
                int prev = colidx[p - 1];
                if (c == prev) f |= F_DUPLICATE;
                else if (c < prev) f |= F_UNSORTED;
            }
        }
    }
    f = __reduce_or_sync(0xffffffffu, f);
    if (lane == 0 && f) atomicOr(flags, f);
}

// ---------------------------------------------------------------- F1 (sort path)
// Output per window: u[w] (unique count), nb[w] = ceil(u/8), uniq[s0 + k] (k < u)
// ascending unique columns, rank[p] for p in the segment.
template <int WH>
__global__ void __launch_bounds__(kSortThreads)
k_dedup_sort(int64_t M, int64_t K, int64_t nnz, const int32_t* __restrict__ rowptr,
             const int32_t* __restrict__ colidx, int mode, int32_t* __restrict__ u_out,
             int64_t* __restrict__ nb_out, int32_t* __restrict__ uniq, int32_t* __restrict__ rank) {
    __shared__ int s_key[kSortMax];
    __shared__ int s_u[kSortMax];
    const int64_t w = blockIdx.x;
    int64_t s0, s1;
    window_segment<WH>(rowptr, M, nnz, w, &s0, &s1);
    const int64_t n64 = s1 - s0;
    const int n = n64 > INT_MAX ? INT_MAX : (int)n64;
    if (n > kSortMax || mode == 2) return;  // bitmap path handles it
    if (n == 0) {
        if (threadIdx.x == 0) { u_out[w] = 0; nb_out[w] = 0; }
        return;
    }
    int P = 32;
    while (P < n) P <<= 1;
    for (int i = threadIdx.x; i < P; i += kSortThreads) s_key[i] = i < n ? colidx[s0 + i] : INT_MAX;
    __syncthreads();
    for (int k = 2; k <= P; k <<= 1) {
        for (int j = k >> 1; j > 0; j >>= 1) {
            for (int i = threadIdx.x; i < P; i += kSortThreads) {
                int ixj = i ^ j;
                if (ixj > i) {
                    int a = s_key[i], b = s_key[ixj];
                    bool up = (i & k) == 0;
                    if ((a > b) == up) { s_key[i] = b; s_key[ixj] = a; }
                }
            }
            __syncthreads();
        }
    }
    // unique compaction: each thread owns a contiguous run of ITEMS keys
    constexpr int ITEMS = kSortMax / kSortThreads;
    const int i0 = threadIdx.x * ITEMS;
    int cnt = 0;
#pragma unroll
    for (int q = 0; q < ITEMS; ++q) {
        int i = i0 + q;
        if (i < n && (i == 0 || s_key[i] != s_key[i - 1])) ++cnt;
    }
    int total;
    int pos = block_exscan<kSortThreads>(cnt, &total);
#pragma unroll
    for (int q = 0; q < ITEMS; ++q) {
        int i = i0 + q;
        if (i < n && (i == 0 || s_key[i] != s_key[i - 1])) {
            s_u[pos] = s_key[i];
            uniq[s0 + pos] = s_key[i];
            ++pos;
        }
    }
    __syncthreads();
    for (int i = threadIdx.x; i < n; i += kSortThreads) {
        int c = colidx[s0 + i];
        int lo = 0, hi = total;
        while (lo < hi) {
            int mid = (lo + hi) >> 1;
            if (s_u[mid] < c) lo = mid + 1; else hi = mid;
        }
        rank[s0 + i] = lo;
    }
    if (threadIdx.x == 0) {
        u_out[w] = total;
        nb_out[w] = (total + kTcw - 1) / kTcw;
    }
}

// ---------------------------------------------------------------- F1 (bitmap path)
template <int WH>
__global__ void __launch_bounds__(kBmThreads)
k_dedup_bitmap(int64_t M, int64_t K, int64_t nnz, const int32_t* __restrict__ rowptr,
               const int32_t* __restrict__ colidx, int mode, int32_t* __restrict__ u_out,
               int64_t* __restrict__ nb_out, int32_t* __restrict__ uniq, int32_t* __restrict__ rank) {
    extern __shared__ uint32_t smem_bm[];
    uint32_t* bm = smem_bm;                 // [kBmWords]
    int* pref = (int*)(smem_bm + kBmWords); // [kBmWords] exclusive popcount prefix
    const int64_t w = blockIdx.x;
    int64_t s0, s1;
    window_segment<WH>(rowptr, M, nnz, w, &s0, &s1);
    const int64_t n = s1 - s0;
    if (mode != 2 && n <= kSortMax) return;  // sort path handled it
    int lo = INT_MAX, hi = -1;
    for (int64_t p = s0 + threadIdx.x; p < s1; p += kBmThreads) {
        int c = colidx[p];
        if (c >= 0 && c < K) { lo = min(lo, c); hi = max(hi, c); }
    }
    lo = block_min<kBmThreads>(lo);
    hi = block_max<kBmThreads>(hi);
    int64_t base_rank = 0;
    constexpr int WPT = kBmWords / kBmThreads;  // words per thread in the scan
    for (int64_t c0 = lo; c0 <= hi; c0 += kBmBits) {
        for (int i = threadIdx.x; i < kBmWords; i += kBmThreads) bm[i] = 0u;
        __syncthreads();
        for (int64_t p = s0 + threadIdx.x; p < s1; p += kBmThreads) {
            int64_t c = colidx[p];
            if (c >= c0 && c < c0 + kBmBits && c < K) {
                int off = (int)(c - c0);
                atomicOr(&bm[off >> 5], 1u << (off & 31));
            }
        }
        __syncthreads();
        int my = 0;
        const int wb = threadIdx.x * WPT;
#pragma unroll 8
        for (int q = 0; q < WPT; ++q) my += __popc(bm[wb + q]);
        int chunk_total;
        int run = block_exscan<kBmThreads>(my, &chunk_total);
        for (int q = 0; q < WPT; ++q) {
            uint32_t bits = bm[wb + q];
            pref[wb + q] = run;
            int k = 0;
            while (bits) {
                int b = __ffs(bits) - 1;
                bits &= bits - 1;
                uniq[s0 + base_rank + run + k] = (int32_t)(c0 + (int64_t)(wb + q) * 32 + b);
                ++k;
            }
            run += k;
        }
        __syncthreads();
        for (int64_t p = s0 + threadIdx.x; p < s1; p += kBmThreads) {
            int64_t c = colidx[p];
            if (c >= c0 && c < c0 + kBmBits && c < K) {
                int off = (int)(c - c0);
                uint32_t word = bm[off >> 5];
                rank[p] = (int32_t)(base_rank + pref[off >> 5] +
                                    __popc(word & ((1u << (off & 31)) - 1u)));
            }
        }
        base_rank += chunk_total;
        __syncthreads();
    }
    if (threadIdx.x == 0) {
        u_out[w] = (int32_t)base_rank;
        nb_out[w] = (base_rank + kTcw - 1) / kTcw;
    }
}

// ---------------------------------------------------------------- optional row permutation
// (dtc_build_opts_t.row_perm, e.g. the TCA order): check it is a bijection, then gather the
// permuted CSR (new row r = original row perm[r]) that F0-F4 then condense.
__global__ void k_perm_count(int64_t M, const int32_t* __restrict__ perm, int32_t* __restrict__ seen,
                             int* __restrict__ flags) {
    for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < M; r += (int64_t)gridDim.x * blockDim.x) {
        const int32_t v = perm[r];
        if (v < 0 || v >= M) atomicOr(flags, 1);
        else atomicAdd(&seen[v], 1);
    }
}
__global__ void k_perm_deg(int64_t M, const int32_t* __restrict__ perm, const int32_t* __restrict__ seen,
                           const int32_t* __restrict__ rowptr, int64_t nnz, int64_t* __restrict__ deg,
                           int* __restrict__ flags) {
    for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < M; r += (int64_t)gridDim.x * blockDim.x) {
        if (seen[r] != 1) atomicOr(flags, 1);
        int64_t v = perm[r];
        v = v < 0 ? 0 : (v >= M ? M - 1 : v);
        const int64_t a = clamp64(rowptr[v], 0, nnz), b = clamp64(rowptr[v + 1], 0, nnz);
        deg[r] = b > a ? b - a : 0;
    }
}
template <class V>
__global__ void k_perm_copy(int64_t M, const int32_t* __restrict__ perm, const int32_t* __restrict__ rowptr,
                            const int64_t* __restrict__ nrp, const int32_t* __restrict__ ci, const V* __restrict__ vi,
                            int32_t* __restrict__ co, V* __restrict__ vo) {
    const int lane = threadIdx.x & 31;
    int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t r = warp; r < M; r += nwarps) {
        int64_t v = perm[r];
        v = v < 0 ? 0 : (v >= M ? M - 1 : v);
        const int64_t src = rowptr[v], dst = nrp[r], n = nrp[r + 1] - nrp[r];
        for (int64_t k = lane; k < n; k += 32) {
            co[dst + k] = ci[src + k];
            vo[dst + k] = vi[src + k];
        }
    }
}

// ---------------------------------------------------------------- optional transpose
// (dtc_build_opts_t.transpose): the ME-TCF of A^T -- e.g. for the GCN backward dH = A^T dAH -- from
// A's CSR on the GPU: one 64-bit key (column << rbits | row) per non-zero, a radix sort (CUB, a
// plain library sort of the one-time build) keyed by (column, row) gives A^T's canonical CSR
// (rows = A's columns, entries by ascending original row), values gathered by the sorted index.
__global__ void k_tr_keys(int64_t M, int64_t nnz, const int32_t* __restrict__ rowptr, const int32_t* __restrict__ ci,
                          int rbits, uint64_t* __restrict__ keys, int32_t* __restrict__ idx) {
    const int lane = threadIdx.x & 31;
    int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t r = warp; r < M; r += nwarps) {
        const int64_t lo = clamp64(rowptr[r], 0, nnz), hi = clamp64(rowptr[r + 1], 0, nnz);
        for (int64_t p = lo + lane; p < hi; p += 32) {
            keys[p] = ((uint64_t)(uint32_t)ci[p] << rbits) | (uint64_t)r;
            idx[p] = (int32_t)p;
        }
    }
}
template <class V>
__global__ void k_tr_fill(int64_t nnz, int64_t Mt, int rbits, const uint64_t* __restrict__ keys,
                          const int32_t* __restrict__ idx, const V* __restrict__ vin, int32_t* __restrict__ rowptr_t,
                          int32_t* __restrict__ ci_t, V* __restrict__ v_t) {
    const uint64_t rmask = (uint64_t(1) << rbits) - 1;
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e <= nnz; e += (int64_t)gridDim.x * blockDim.x) {
        // row c of A^T starts at the first sorted key of column c: fill rowptr_t[prev+1 .. c]
        const int64_t c = e < nnz ? (int64_t)(keys[e] >> rbits) : Mt;
        const int64_t prev = e > 0 ? (int64_t)(keys[e - 1] >> rbits) : -1;
        for (int64_t k = prev + 1; k <= c; ++k) rowptr_t[k] = (int32_t)e;
        if (e < nnz) {
            ci_t[e] = (int32_t)(keys[e] & rmask);
            v_t[e] = vin[idx[e]];
        }
    }
}

// ---------------------------------------------------------------- F2/F3
__global__ void k_to_i32(const int64_t* __restrict__ in, int32_t* __restrict__ out, int64_t n) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = (int32_t)in[i];
}

// F3, one CTA per window (no global atomics for windows of <= kFillSmemBlocks TC blocks):
//   SparseAtoB[8*(b0+j) + i] = U[8j + i] (or -1);  a 128-bit occupancy mask per block (bit =
//   local id) built with shared-memory atomics; TCOffset by a CTA scan of the masks' popcounts
//   starting at rowptr[16w] (= TCOffset[RWO[w]]); every nnz then lands at
//   TCOffset[b] + popcount(mask[b] below its id) -- ascending local id inside a block (C5).
constexpr int kFillThreads = 256;
constexpr int kFillSmemBlocks = 1024;

template <class V, int WH>
__global__ void __launch_bounds__(kFillThreads)
k_fill_window(int64_t W, int64_t M, int64_t nnz, const int32_t* __restrict__ rowptr, const int32_t* __restrict__ rwo,
              const int32_t* __restrict__ u, const int32_t* __restrict__ uniq, const int32_t* __restrict__ rank,
              uint32_t* __restrict__ gmask, const V* __restrict__ vin, int32_t* __restrict__ tco,
              uint8_t* __restrict__ lid, V* __restrict__ vout, int32_t* __restrict__ atob) {
    constexpr int MW = WH * kTcw / 32;   // mask words per block: one bit per local id (128 or 256)
    __shared__ uint32_t s_mask[kFillSmemBlocks * MW];
    __shared__ int s_off[kFillSmemBlocks];
    __shared__ int s_rp[WH + 1];
    const int tid = threadIdx.x;
    const int64_t w = blockIdx.x;
    int64_t s0, s1;
    window_segment<WH>(rowptr, M, nnz, w, &s0, &s1);
    const int64_t r0 = w * WH;
    const int nrows = (M - r0) < WH ? (int)(M - r0) : WH;
    const int64_t b0 = rwo[w];
    const int nb = (int)(rwo[w + 1] - b0);
    const bool sm = nb <= kFillSmemBlocks;
    uint32_t* mask = sm ? s_mask : gmask + b0 * MW;
    if (tid <= nrows) s_rp[tid] = (int)clamp64(rowptr[r0 + tid], s0, s1);
    if (sm) for (int i = tid; i < nb * MW; i += kFillThreads) s_mask[i] = 0u;
    const int uw = u[w];
    for (int64_t k = tid; k < (int64_t)nb * kTcw; k += kFillThreads)
        atob[b0 * kTcw + k] = k < uw ? uniq[s0 + k] : -1;
    __syncthreads();
    auto row_of = [&](int64_t p) {   // s_rp[r] <= p < s_rp[r+1]
        int lo = 0, hi = nrows;
        while (hi - lo > 1) {
            const int mid = (lo + hi) >> 1;
            if (s_rp[mid] <= p) lo = mid; else hi = mid;
        }
        return lo;
    };
    for (int64_t p = s0 + tid; p < s1; p += kFillThreads) {
        const int r = row_of(p);
        const int k = rank[p];
        const int id = r * kTcw + (k & 7);
        atomicOr(&mask[(k >> 3) * MW + (id >> 5)], 1u << (id & 31));
    }
    __syncthreads();
    auto mask_word = [&](int j, int q) -> uint32_t { return sm ? s_mask[j * MW + q] : __ldcg(mask + j * MW + q); };
    int64_t running = s0;
    for (int jb = 0; jb < nb; jb += kFillThreads) {
        const int j = jb + tid;
        int c = 0;
        if (j < nb)
#pragma unroll
            for (int q = 0; q < MW; ++q) c += __popc(mask_word(j, q));
        int tot;
        const int ex = block_exscan<kFillThreads>(c, &tot);
        if (j < nb) {
            tco[b0 + j] = (int32_t)(running + ex);
            if (sm) s_off[j] = (int)(running + ex);
        }
        running += tot;
    }
    if (w == W - 1 && tid == 0) tco[b0 + nb] = (int32_t)nnz;
    __syncthreads();
    for (int64_t p = s0 + tid; p < s1; p += kFillThreads) {
        const int r = row_of(p);
        const int k = rank[p];
        const int j = k >> 3;
        const int id = r * kTcw + (k & 7);
        int below = 0;
#pragma unroll
        for (int q = 0; q < MW; ++q) {
            const int lo = q * 32;
            const uint32_t m = mask_word(j, q);
            if (id >= lo + 32) below += __popc(m);
            else if (id > lo) below += __popc(m & ((1u << (id - lo)) - 1u));
        }
        const int64_t pos = (int64_t)(sm ? s_off[j] : __ldcg(tco + b0 + j)) + below;
        lid[pos] = (uint8_t)id;
        vout[pos] = vin[p];
    }
    if (sm)   // persist the masks (the kernel-side fragment index)
        for (int i = tid; i < nb * MW; i += kFillThreads) gmask[b0 * MW + i] = s_mask[i];
}

// ---------------------------------------------------------------- F4
// F4 rules (Guide, split_pieces): dtc_sched.h, shared with the Selector's host simulation.

__global__ void k_units_count(int64_t W, const int32_t* __restrict__ rwo, Guide gd,
                              int64_t* __restrict__ cnt, int64_t* __restrict__ split,
                              int64_t* __restrict__ slots) {
    for (int64_t w = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; w < W; w += (int64_t)gridDim.x * blockDim.x) {
        const int64_t nb = rwo[w + 1] - rwo[w];
        const int64_t U = gd.size_at(rwo[w]);
        const bool big = nb > U;
        int64_t c;
        if (big) {
            c = split_pieces(nb, U);
        } else {
            bool starts = (w == 0);
            if (!starts) {
                const int64_t pnb = rwo[w] - rwo[w - 1];
                starts = (pnb > gd.size_at(rwo[w - 1])) || (gd.chunk(rwo[w]) != gd.chunk(rwo[w - 1]));
            }
            c = starts ? 1 : 0;
        }
        cnt[w] = c;
        split[w] = big ? 1 : 0;
        slots[w] = big ? c : 0;
    }
}

__global__ void k_units_fill(int64_t W, const int32_t* __restrict__ rwo, Guide gd,
                             const int64_t* __restrict__ ubase, const int64_t* __restrict__ sbase,
                             const int64_t* __restrict__ slbase, Unit* __restrict__ units) {
    for (int64_t w = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; w < W; w += (int64_t)gridDim.x * blockDim.x) {
        int64_t c = ubase[w + 1] - ubase[w];
        if (c == 0) continue;
        int64_t nb = rwo[w + 1] - rwo[w];
        if (nb > gd.size_at(rwo[w])) {
            for (int64_t p = 0; p < c; ++p) {
                Unit u;
                u.wb = (int32_t)w; u.we = (int32_t)(w + 1);
                u.bb = (int32_t)(rwo[w] + p * nb / c);
                u.be = (int32_t)(rwo[w] + (p + 1) * nb / c);
                u.split_id = (int32_t)sbase[w]; u.piece = (int32_t)p; u.npieces = (int32_t)c;
                u.slot_base = (int32_t)slbase[w];
                units[ubase[w] + p] = u;
            }
        } else {
            Unit u;
            u.wb = (int32_t)w; u.we = -1; u.bb = rwo[w]; u.be = -1;
            u.split_id = -1; u.piece = 0; u.npieces = 1; u.slot_base = 0;
            units[ubase[w]] = u;
        }
    }
}

__global__ void k_units_fix(int64_t nu, int64_t W, const int32_t* __restrict__ rwo, Unit* __restrict__ units) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nu; i += (int64_t)gridDim.x * blockDim.x) {
        if (units[i].split_id >= 0) continue;
        int64_t we = (i + 1 < nu) ? units[i + 1].wb : W;
        units[i].we = (int32_t)we;
        units[i].be = rwo[we];
    }
}

// Unit order: the pieces of split windows first (window order among them), then the whole-window
// units (window order).  The last-arriving piece of a split window sums all its partials -- a chain
// of npieces dependent loads -- so those units go first, where their fixups overlap the rest of the
// launch instead of forming its tail (longest-processing-time-first).  Results do not depend on
// the order (each unit is computed the same way; partials are summed in piece order).
__global__ void k_units_flag(int64_t nu, const Unit* __restrict__ units, int64_t* __restrict__ flag) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nu; i += (int64_t)gridDim.x * blockDim.x)
        flag[i] = units[i].split_id >= 0 ? 1 : 0;
}
__global__ void k_units_permute(int64_t nu, const Unit* __restrict__ in, const int64_t* __restrict__ pos,
                                Unit* __restrict__ out) {
    const int64_t nsu = pos[nu];
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nu; i += (int64_t)gridDim.x * blockDim.x) {
        const bool sp = in[i].split_id >= 0;
        out[sp ? pos[i] : nsu + (i - pos[i])] = in[i];
    }
}

// ---------------------------------------------------------------- host driver
static unsigned grid_for(int64_t work, int per_block, int cap = 1 << 20) {
    int64_t g = (work + per_block - 1) / per_block;
    if (g < 1) g = 1;
    if (g > cap) g = cap;
    return (unsigned)g;
}

static void free_format(dtc_format* h, cudaStream_t s) {
    if (!h) return;
    dfree(h->rwo, s); dfree(h->tco, s); dfree(h->lid, s); dfree(h->atob, s);
    dfree(h->vals, s); dfree(h->mask, s); dfree(h->units, s); dfree(h->counters, s); dfree(h->ws, s);
    for (auto& e : h->hev) if (e) { cudaEventDestroy(e); e = nullptr; }
    for (auto& hs : h->hstream) if (hs) { cudaStreamDestroy(hs); hs = nullptr; }
    for (int k = 0; k < 2; ++k) {
        dfree(h->as_B[k], s); dfree(h->as_C[k], s);
        if (h->as_ev_in[k]) cudaEventDestroy(h->as_ev_in[k]);
        if (h->as_ev_kernel[k]) cudaEventDestroy(h->as_ev_kernel[k]);
        if (h->as_ev_out[k]) cudaEventDestroy(h->as_ev_out[k]);
    }
    if (h->as_in) cudaStreamDestroy(h->as_in);
    if (h->as_out) cudaStreamDestroy(h->as_out);
    dfree(h->stage_B, s); dfree(h->stage_C, s); dfree(h->rowmap, s); dfree(h->gemm_ws, s); dfree(h->uctr, s); dfree(h->units_lpt, s); dfree(h->ufirst, s);
}

struct BuildTemps {
    int* flags = nullptr;
    int32_t* u = nullptr;
    int64_t* nb = nullptr;       // [W+1]  -> scanned in place to block offsets
    int32_t* uniq = nullptr;     // [nnz]
    int32_t* rank = nullptr;     // [nnz]
    int64_t* scan_tmp = nullptr;
    int64_t* cnt = nullptr;      // [T+1]
    int64_t* ucnt = nullptr;     // [W+1]
    int64_t* usplit = nullptr;   // [W+1]
    int64_t* uslots = nullptr;   // [W+1]
    int64_t* host = nullptr;     // pinned readback
    int32_t* pseen = nullptr;    // row_perm: hit counts per original row
    int64_t* pdeg = nullptr;     // row_perm: permuted degrees -> rowptr (int64)
    int32_t* prow32 = nullptr;   // row_perm: permuted rowptr
    int32_t* pcol = nullptr;     // row_perm: permuted colidx
    uint8_t* pval = nullptr;     // row_perm: permuted values
    uint64_t* tkeys = nullptr;   // transpose: sort keys (in / out)
    uint64_t* tkeys2 = nullptr;
    int32_t* tidx = nullptr;     // transpose: nnz index (in / out)
    int32_t* tidx2 = nullptr;
    uint8_t* tsort = nullptr;    // transpose: CUB temp storage
    void release(cudaStream_t s) {
        dfree(tkeys, s); dfree(tkeys2, s); dfree(tidx, s); dfree(tidx2, s); dfree(tsort, s);
        dfree(flags, s); dfree(u, s); dfree(nb, s); dfree(uniq, s); dfree(rank, s);
        dfree(scan_tmp, s); dfree(cnt, s); dfree(ucnt, s); dfree(usplit, s);
        dfree(uslots, s);
        dfree(pseen, s); dfree(pdeg, s); dfree(prow32, s); dfree(pcol, s); dfree(pval, s);
        host = nullptr;   // per-thread pinned scratch, not owned
    }
};

// F4 unit size: ~2 windows' worth of TC blocks, clamped to [64, 256] (measured sweep for the
// TMA path, profiles/r01_design_evidence.md: arxiv-like 64, banded 64-128, products-like 128,
// reddit-like >= 256), and small enough for >= 4 waves of 6 CTAs per SM (so the last partial wave
// is a small part of the launch: arxiv-like T = 115k -> U = 32, +3% measured over U = 64 in three
// runs); never below 16.
static int auto_unit_blocks(int64_t T, int64_t W) {
    int64_t target = W > 0 ? (2 * T) / W : 64;
    if (target < 64) target = 64;
    if (target > 256) target = 256;
    const int64_t cap = T / (24 * (int64_t)num_sms());
    if (target > cap) target = cap < 16 ? 16 : cap;
    return (int)target;
}

// DTC_BUILD_PROFILE=1: synchronise and print the wall time of each build stage (diagnostics only).
struct StageTimer {
    bool on = false;
    cudaStream_t s = nullptr;
    std::chrono::steady_clock::time_point t0;
    void init(cudaStream_t st) {
        const char* e = getenv("DTC_BUILD_PROFILE");
        on = e && e[0] == '1';
        s = st;
        if (on) { cudaStreamSynchronize(s); t0 = std::chrono::steady_clock::now(); }
    }
    void mark(const char* what) {
        if (!on) return;
        cudaStreamSynchronize(s);
        auto t1 = std::chrono::steady_clock::now();
        fprintf(stderr, "[dtc build] %-28s %9.3f ms\n", what, std::chrono::duration<double, std::milli>(t1 - t0).count());
        t0 = t1;
    }
};

int format_build(const dtc_csr_t* csr, const dtc_build_opts_t* opts, cudaStream_t s, dtc_format** out) {
    if (!out) { set_error("out is NULL"); return DTC_ERR_INVALID; }
    *out = nullptr;
    if (!csr) { set_error("csr is NULL"); return DTC_ERR_INVALID; }
    const int64_t M = csr->M, K = csr->K, nnz = csr->nnz;
    if (M < 0 || K < 0 || nnz < 0 || nnz >= INT32_MAX || M >= INT32_MAX - 16 || K >= INT32_MAX) {
        set_error("bad sizes M=%lld K=%lld nnz=%lld", (long long)M, (long long)K, (long long)nnz);
        return DTC_ERR_INVALID;
    }
    if (csr->dtype != DTC_TF32 && csr->dtype != DTC_FP16) { set_error("bad dtype %d", csr->dtype); return DTC_ERR_INVALID; }
    if (!csr->rowptr || (nnz > 0 && (!csr->colidx || !csr->vals))) { set_error("null CSR pointer"); return DTC_ERR_INVALID; }
    if (M == 0 && nnz != 0) { set_error("M == 0 but nnz != 0"); return DTC_ERR_INVALID; }
    int dev_count = 0;
    if (cudaGetDeviceCount(&dev_count) != cudaSuccess || dev_count == 0) {
        cudaGetLastError();
        set_error("no CUDA device");
        return DTC_ERR_CUDA;
    }
    const int mode = opts ? opts->dedup_path : 0;
    const bool transpose = opts && opts->transpose;
    if (transpose && opts->row_perm) { set_error("transpose and row_perm cannot be combined"); return DTC_ERR_INVALID; }
    // the condensed matrix: A (M x K) or A^T (K x M)
    const int64_t Mc = transpose ? K : M, Kc = transpose ? M : K;
    int WH = (opts && opts->window_rows > 0) ? opts->window_rows : kWindow;
    if (WH != 16 && WH != 32) { set_error("window_rows must be 16 or 32"); return DTC_ERR_INVALID; }
    // Selector, window height (NEXT-2): 32-row windows pay when two 16-row windows share >= 35% of
    // their gathered B rows (T32 <= 0.65 T16) and each gathered row is >= 1 KB, so the saved bytes
    // outweigh the doubled MMA / fragment work (c4 N=256: +17%; every other workload loses;
    // profiles/r02_ab_tall_windows.txt).  TF32 only; needs F0-F2 at both heights (two extra passes).
    if (opts && opts->selector > 0 && opts->window_rows == 0 && csr->dtype == DTC_TF32 && !transpose &&
        !opts->row_perm && (int64_t)(opts->n_hint > 0 ? opts->n_hint : 128) * 4 >= 1024 && csr->nnz > 0) {
        std::vector<int32_t> r16, r32;
        int rc0 = window_offsets(csr, s, &r16, 16);
        if (rc0 == DTC_OK) rc0 = window_offsets(csr, s, &r32, 32);
        if (rc0 != DTC_OK) return rc0;
        const double t16 = (double)r16.back(), t32 = (double)r32.back();
        if (t16 > 0 && t32 <= 0.65 * t16) WH = 32;
    }
    if (WH == 32 && csr->dtype != DTC_TF32) { set_error("window_rows = 32 is implemented for TF32"); return DTC_ERR_UNSUPPORTED; }
    const int64_t W = (Mc + WH - 1) / WH;

    dtc_format* h = new (std::nothrow) dtc_format();
    if (!h) { set_error("host OOM"); return DTC_ERR_OOM; }
    h->M = Mc; h->K = Kc; h->nnz = nnz; h->W = W; h->dtype = csr->dtype; h->window_h = WH;
    cudaGetDevice(&h->device);
    BuildTemps t;
    dtc_csr_t pcsr;   // permuted CSR view (row_perm)
    StageTimer st;
    st.init(s);
    int rc = DTC_OK;
#define TRY(x) do { rc = (x); if (rc != DTC_OK) goto fail; } while (0)
#define TRYC(x) do { cudaError_t _e = (x); if (_e != cudaSuccess) { rc = cuda_fail(_e, #x, __FILE__, __LINE__); goto fail; } } while (0)
    {
        t.host = pinned_scratch();
        if (!t.host) { set_error("pinned host scratch allocation failed"); rc = DTC_ERR_OOM; goto fail; }
        TRY(dalloc(&t.flags, 1, s));
        TRYC(cudaMemsetAsync(t.flags, 0, sizeof(int), s));
        TRY(dalloc(&t.u, W + 1, s));
        TRY(dalloc(&t.nb, W + 1, s));
        TRY(dalloc(&t.uniq, nnz, s));
        TRY(dalloc(&t.rank, nnz, s));
        const int64_t scan_n = std::max<int64_t>(W + 1, 1);
        if (opts && opts->row_perm && M > 0) {
            // permuted CSR (F0 below validates its columns; the bijection is checked here)
            TRY(dalloc(&t.pseen, M, s));
            TRYC(cudaMemsetAsync(t.pseen, 0, M * sizeof(int32_t), s));
            TRY(dalloc(&t.pdeg, M + 1, s));
            TRY(dalloc(&t.scan_tmp, scan_tmp_elems(M + 1) + 64, s));
            TRY(dalloc(&t.prow32, M + 1, s));
            TRY(dalloc(&t.pcol, nnz, s));
            TRY(dalloc(&t.pval, (size_t)std::max<int64_t>(nnz, 1) * elt_size(h->dtype), s));
            k_perm_count<<<grid_for(M, 256, 4096), 256, 0, s>>>(M, opts->row_perm, t.pseen, t.flags);
            k_perm_deg<<<grid_for(M, 256, 4096), 256, 0, s>>>(M, opts->row_perm, t.pseen, csr->rowptr, nnz, t.pdeg, t.flags);
            exclusive_scan_i64(t.pdeg, t.pdeg, M, t.scan_tmp, s);
            k_to_i32<<<grid_for(M + 1, 256, 4096), 256, 0, s>>>(t.pdeg, t.prow32, M + 1);
            if (h->dtype == DTC_FP16)
                k_perm_copy<uint16_t><<<grid_for(M * 32, 256, 148 * 64), 256, 0, s>>>(
                    M, opts->row_perm, csr->rowptr, t.pdeg, csr->colidx, (const uint16_t*)csr->vals, t.pcol,
                    (uint16_t*)t.pval);
            else
                k_perm_copy<uint32_t><<<grid_for(M * 32, 256, 148 * 64), 256, 0, s>>>(
                    M, opts->row_perm, csr->rowptr, t.pdeg, csr->colidx, (const uint32_t*)csr->vals, t.pcol,
                    (uint32_t*)t.pval);
            TRY(dalloc(&h->rowmap, M, s));
            TRYC(cudaMemcpyAsync(h->rowmap, opts->row_perm, M * sizeof(int32_t), cudaMemcpyDeviceToDevice, s));
            dfree(t.scan_tmp, s);
            pcsr = *csr;
            pcsr.rowptr = t.prow32;
            pcsr.colidx = t.pcol;
            pcsr.vals = t.pval;
            csr = &pcsr;
        }
        if (transpose && nnz > 0) {
            // validate A itself (its keys must be in range), then build A^T's CSR and condense that
            k_validate<<<grid_for(M * 32, 256, 148 * 64), 256, 0, s>>>(M, K, nnz, csr->rowptr, csr->colidx, t.flags);
            TRYC(cudaMemcpyAsync(&t.host[1], t.flags, sizeof(int), cudaMemcpyDeviceToHost, s));
            TRYC(cudaStreamSynchronize(s));
            const int f0 = (int)(t.host[1] & 0xffffffff);
            if (f0) {
                if (f0 & F_INVALID) { set_error("malformed rowptr"); rc = DTC_ERR_INVALID; }
                else if (f0 & F_RANGE) { set_error("column index out of [0, K)"); rc = DTC_ERR_RANGE; }
                else if (f0 & F_DUPLICATE) { set_error("duplicate column within a row"); rc = DTC_ERR_DUPLICATE; }
                else { set_error("columns not ascending within a row"); rc = DTC_ERR_UNSORTED; }
                goto fail;
            }
            int rbits = 1;
            while ((int64_t(1) << rbits) < M) ++rbits;
            int cbits = 1;
            while ((int64_t(1) << cbits) < K) ++cbits;
            TRY(dalloc(&t.tkeys, nnz, s));
            TRY(dalloc(&t.tkeys2, nnz, s));
            TRY(dalloc(&t.tidx, nnz, s));
            TRY(dalloc(&t.tidx2, nnz, s));
            k_tr_keys<<<grid_for(M * 32, 256, 148 * 64), 256, 0, s>>>(M, nnz, csr->rowptr, csr->colidx, rbits, t.tkeys, t.tidx);
            size_t tb = 0;
            TRYC(cub::DeviceRadixSort::SortPairs(nullptr, tb, t.tkeys, t.tkeys2, t.tidx, t.tidx2, (int)nnz, 0,
                                                 rbits + cbits, s));
            TRY(dalloc(&t.tsort, tb, s));
            TRYC(cub::DeviceRadixSort::SortPairs(t.tsort, tb, t.tkeys, t.tkeys2, t.tidx, t.tidx2, (int)nnz, 0,
                                                 rbits + cbits, s));
            TRY(dalloc(&t.prow32, Mc + 1, s));
            TRY(dalloc(&t.pcol, nnz, s));
            TRY(dalloc(&t.pval, (size_t)nnz * elt_size(h->dtype), s));
            if (h->dtype == DTC_FP16)
                k_tr_fill<uint16_t><<<grid_for(nnz + 1, 256, 148 * 64), 256, 0, s>>>(
                    nnz, Mc, rbits, t.tkeys2, t.tidx2, (const uint16_t*)csr->vals, t.prow32, t.pcol, (uint16_t*)t.pval);
            else
                k_tr_fill<uint32_t><<<grid_for(nnz + 1, 256, 148 * 64), 256, 0, s>>>(
                    nnz, Mc, rbits, t.tkeys2, t.tidx2, (const uint32_t*)csr->vals, t.prow32, t.pcol, (uint32_t*)t.pval);
            TRYC(cudaGetLastError());
            dfree(t.tkeys, s); dfree(t.tkeys2, s); dfree(t.tidx, s); dfree(t.tidx2, s); dfree(t.tsort, s);
            pcsr = *csr;
            pcsr.M = Mc; pcsr.K = Kc;
            pcsr.rowptr = t.prow32;
            pcsr.colidx = t.pcol;
            pcsr.vals = t.pval;
            csr = &pcsr;
        } else if (transpose) {
            TRY(dalloc(&t.prow32, Mc + 1, s));
            TRYC(cudaMemsetAsync(t.prow32, 0, (Mc + 1) * sizeof(int32_t), s));
            pcsr = *csr;
            pcsr.M = Mc; pcsr.K = Kc;
            pcsr.rowptr = t.prow32;
            csr = &pcsr;
        }
        st.mark("setup+temp alloc");
        // F0
        if (Mc > 0) k_validate<<<grid_for(Mc * 32, 256, 148 * 64), 256, 0, s>>>(Mc, Kc, nnz, csr->rowptr, csr->colidx, t.flags);
        st.mark("F0 validate");
        // F1
        if (W > 0) {
            const size_t bm_smem = 2 * kBmWords * sizeof(uint32_t);
            if (WH == 16) {
                k_dedup_sort<16><<<(unsigned)W, kSortThreads, 0, s>>>(Mc, Kc, nnz, csr->rowptr, csr->colidx, mode,
                                                                     t.u, t.nb, t.uniq, t.rank);
                TRYC(cudaFuncSetAttribute(k_dedup_bitmap<16>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bm_smem));
                k_dedup_bitmap<16><<<(unsigned)W, kBmThreads, bm_smem, s>>>(Mc, Kc, nnz, csr->rowptr, csr->colidx,
                                                                           mode, t.u, t.nb, t.uniq, t.rank);
            } else {
                k_dedup_sort<32><<<(unsigned)W, kSortThreads, 0, s>>>(Mc, Kc, nnz, csr->rowptr, csr->colidx, mode,
                                                                     t.u, t.nb, t.uniq, t.rank);
                TRYC(cudaFuncSetAttribute(k_dedup_bitmap<32>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bm_smem));
                k_dedup_bitmap<32><<<(unsigned)W, kBmThreads, bm_smem, s>>>(Mc, Kc, nnz, csr->rowptr, csr->colidx,
                                                                           mode, t.u, t.nb, t.uniq, t.rank);
            }
        }
        TRYC(cudaGetLastError());
        st.mark("F1 dedup");
        // F2: RowWindowOffset = exclusive scan of nTC_w
        TRY(dalloc(&t.scan_tmp, scan_tmp_elems(scan_n) + 64, s));
        if (W > 0) exclusive_scan_i64(t.nb, t.nb, W, t.scan_tmp, s);
        else TRYC(cudaMemsetAsync(t.nb, 0, sizeof(int64_t), s));
        TRYC(cudaMemcpyAsync(&t.host[0], t.nb + W, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
        TRYC(cudaMemcpyAsync(&t.host[1], t.flags, sizeof(int), cudaMemcpyDeviceToHost, s));
        TRYC(cudaStreamSynchronize(s));  // host sync #1: T and the validation flag
        const int64_t T = t.host[0];
        const int flags = (int)(t.host[1] & 0xffffffff);
        if (flags) {
            if (flags & F_INVALID) { set_error("malformed rowptr"); rc = DTC_ERR_INVALID; }
            else if (flags & F_RANGE) { set_error("column index out of [0, K)"); rc = DTC_ERR_RANGE; }
            else if (flags & F_DUPLICATE) { set_error("duplicate column within a row"); rc = DTC_ERR_DUPLICATE; }
            else { set_error("columns not ascending within a row"); rc = DTC_ERR_UNSORTED; }
            goto fail;
        }
        if (T >= INT32_MAX / 8) { set_error("NumTCBlock %lld too large for int32 indexing", (long long)T); rc = DTC_ERR_UNSUPPORTED; goto fail; }
        h->T = T;
        st.mark("F2 scan+sync");
        // F3
        TRY(dalloc(&h->rwo, W + 1, s));
        TRY(dalloc(&h->tco, T + 1, s));
        TRY(dalloc(&h->lid, nnz, s));
        TRY(dalloc(&h->atob, 8 * T, s));
        {
            uint8_t* vb = nullptr;
            // +16 bytes: the SpMM TMA path bulk-copies 16-byte aligned supersets of value ranges
            TRY(dalloc(&vb, (size_t)std::max<int64_t>(nnz, 1) * elt_size(h->dtype) + 16, s));
            h->vals = vb;
        }
        k_to_i32<<<grid_for(W + 1, 256, 4096), 256, 0, s>>>(t.nb, h->rwo, W + 1);
        if (T > 0) {
            // occupancy masks: built in shared memory (windows of <= kFillSmemBlocks blocks) or
            // directly in this array, which the SpMM kernel keeps as its fragment index
            const int64_t mw = WH * kTcw / 32;   // mask words per block
            TRY(dalloc(&h->mask, mw * T, s));
            TRYC(cudaMemsetAsync(h->mask, 0, mw * T * sizeof(uint32_t), s));
#define DTC_FILL(V, WHV)                                                                                         \
    k_fill_window<V, WHV><<<(unsigned)W, kFillThreads, 0, s>>>(W, Mc, nnz, csr->rowptr, h->rwo, t.u, t.uniq, t.rank, \
                                                              h->mask, (const V*)csr->vals, h->tco, h->lid,        \
                                                              (V*)h->vals, h->atob)
            if (h->dtype == DTC_FP16) {
                if (WH == 16) DTC_FILL(uint16_t, 16); else DTC_FILL(uint16_t, 32);
            } else {
                if (WH == 16) DTC_FILL(uint32_t, 16); else DTC_FILL(uint32_t, 32);
            }
#undef DTC_FILL
        } else {
            TRYC(cudaMemsetAsync(h->tco, 0, sizeof(int32_t), s));
        }
        TRYC(cudaGetLastError());
        st.mark("F3 fill");
        // F4: work units
        int U = (opts && opts->unit_blocks > 0) ? opts->unit_blocks : auto_unit_blocks(T, W);
        // guided tail (units of U/2 over about half a wave): opts->guided 1 = on, -1 = off, 0 = auto:
        // on when the launch is only a few waves long (< 8 waves of 6 CTAs per SM), where the last
        // partial wave is a large part of it (arxiv-shaped c2: +5% measured; c3-c5 have 20-300 waves)
        const int gopt = opts ? opts->guided : 0;
        bool guided = gopt > 0 || (gopt == 0 && T < (int64_t)8 * 6 * num_sms() * U);
        // B200 Selector (NEXT-4, dtc_selector.cu): with no unit size given, simulate the launch of
        // every candidate plan (U x guided tail) for the expected N and keep the shortest
        const int sel = opts ? opts->selector : 0;
        if (!(opts && opts->unit_blocks > 0) && sel == 1 && T > 0) {
            std::vector<int32_t> hrwo((size_t)W + 1);
            TRYC(cudaMemcpyAsync(hrwo.data(), h->rwo, (W + 1) * sizeof(int32_t), cudaMemcpyDeviceToHost, s));
            TRYC(cudaStreamSynchronize(s));
            dtc_sched_model_t m;
            TRY(sched_model(h->dtype, (opts && opts->n_hint > 0) ? opts->n_hint : 128, &m, WH));
            dtc_plan_t best;
            TRY(selector_plan(hrwo.data(), W, m, nullptr, 0, gopt, nullptr, &best));
            U = best.unit_blocks;
            guided = best.guided != 0;
            h->plan_makespan_ns = best.makespan_ns;
        }
        h->unit_blocks = U;
        h->guided = guided ? 1 : 0;
        const int64_t tail = guided ? (int64_t)num_sms() * 4 * U : 0;
        const Guide gd = make_guide(T, U, tail);
        if (W > 0) {
            TRY(dalloc(&t.ucnt, W + 1, s));
            TRY(dalloc(&t.usplit, W + 1, s));
            TRY(dalloc(&t.uslots, W + 1, s));
            k_units_count<<<grid_for(W, 256, 4096), 256, 0, s>>>(W, h->rwo, gd, t.ucnt, t.usplit, t.uslots);
            dfree(t.scan_tmp, s);
            TRY(dalloc(&t.scan_tmp, scan_tmp_elems(W + 1) + 64, s));
            exclusive_scan_i64(t.ucnt, t.ucnt, W, t.scan_tmp, s);
            exclusive_scan_i64(t.usplit, t.usplit, W, t.scan_tmp, s);
            exclusive_scan_i64(t.uslots, t.uslots, W, t.scan_tmp, s);
            TRYC(cudaMemcpyAsync(&t.host[2], t.ucnt + W, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
            TRYC(cudaMemcpyAsync(&t.host[3], t.usplit + W, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
            TRYC(cudaMemcpyAsync(&t.host[4], t.uslots + W, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
            TRYC(cudaStreamSynchronize(s));  // host sync #2: unit count
            h->num_units = t.host[2];
            h->num_split = t.host[3];
            h->num_slots = t.host[4];
            TRY(dalloc(&h->units, std::max<int64_t>(h->num_units, 1), s));
            k_units_fill<<<grid_for(W, 256, 4096), 256, 0, s>>>(W, h->rwo, gd, t.ucnt, t.usplit, t.uslots, h->units);
            k_units_fix<<<grid_for(h->num_units, 256, 4096), 256, 0, s>>>(h->num_units, W, h->rwo, h->units);
            if (h->num_split > 0 && !(opts && opts->window_order)) {
                const int64_t nu = h->num_units;
                int64_t* pos = nullptr;
                Unit* sorted = nullptr;
                TRY(dalloc(&pos, nu + 1, s));
                TRY(dalloc(&sorted, nu, s));
                dfree(t.scan_tmp, s);
                TRY(dalloc(&t.scan_tmp, scan_tmp_elems(nu + 1) + 64, s));
                k_units_flag<<<grid_for(nu, 256, 4096), 256, 0, s>>>(nu, h->units, pos);
                exclusive_scan_i64(pos, pos, nu, t.scan_tmp, s);
                k_units_permute<<<grid_for(nu, 256, 4096), 256, 0, s>>>(nu, h->units, pos, sorted);
                dfree(h->units, s);
                dfree(pos, s);
                h->units = sorted;
            }
        }
        TRYC(cudaGetLastError());
        st.mark("F4 units");
        t.release(s);
        TRYC(cudaStreamSynchronize(s));
        st.mark("release temps");
        *out = h;
        return DTC_OK;
    }
fail:
    cudaGetLastError();
    t.release(s);
    free_format(h, s);
    cudaStreamSynchronize(s);
    delete h;
    return rc;
#undef TRY
#undef TRYC
}

// F0-F2 only: validate the CSR and count each 16-row window's TC blocks, returning RowWindowOffset on
// the host -- all the multi-GPU partitioner needs (no SparseAtoB / values / units are built).
int window_offsets(const dtc_csr_t* csr, cudaStream_t s, std::vector<int32_t>* rwo_out, int WH) {
    if (!csr || !rwo_out) { set_error("null argument"); return DTC_ERR_INVALID; }
    const int64_t M = csr->M, K = csr->K, nnz = csr->nnz;
    if (M < 0 || K < 0 || nnz < 0 || nnz >= INT32_MAX || M >= INT32_MAX - 16 || K >= INT32_MAX || !csr->rowptr ||
        (nnz > 0 && !csr->colidx)) {
        set_error("bad CSR");
        return DTC_ERR_INVALID;
    }
    if (WH != 16 && WH != 32) { set_error("window height %d", WH); return DTC_ERR_INVALID; }
    const int64_t W = (M + WH - 1) / WH;
    int* flags = nullptr;
    int32_t *u = nullptr, *uniq = nullptr, *rank = nullptr;
    int64_t *nb = nullptr, *tmp = nullptr;
    int rc = DTC_OK;
    std::vector<int64_t> h((size_t)W + 1, 0);
    int hflags = 0;
#define TRY(x) do { rc = (x); if (rc != DTC_OK) goto done; } while (0)
#define TRYC(x) do { cudaError_t _e = (x); if (_e != cudaSuccess) { rc = cuda_fail(_e, #x, __FILE__, __LINE__); goto done; } } while (0)
    TRY(dalloc(&flags, 1, s));
    TRYC(cudaMemsetAsync(flags, 0, sizeof(int), s));
    TRY(dalloc(&u, W + 1, s));
    TRY(dalloc(&nb, W + 1, s));
    TRY(dalloc(&uniq, nnz, s));
    TRY(dalloc(&rank, nnz, s));
    TRY(dalloc(&tmp, scan_tmp_elems(W + 1) + 64, s));
    if (M > 0) k_validate<<<grid_for(M * 32, 256, 148 * 64), 256, 0, s>>>(M, K, nnz, csr->rowptr, csr->colidx, flags);
    if (W > 0) {
        const size_t bm_smem = 2 * kBmWords * sizeof(uint32_t);
        if (WH == 16) {
            k_dedup_sort<16><<<(unsigned)W, kSortThreads, 0, s>>>(M, K, nnz, csr->rowptr, csr->colidx, 0, u, nb, uniq, rank);
            TRYC(cudaFuncSetAttribute(k_dedup_bitmap<16>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bm_smem));
            k_dedup_bitmap<16><<<(unsigned)W, kBmThreads, bm_smem, s>>>(M, K, nnz, csr->rowptr, csr->colidx, 0, u, nb,
                                                                       uniq, rank);
        } else {
            k_dedup_sort<32><<<(unsigned)W, kSortThreads, 0, s>>>(M, K, nnz, csr->rowptr, csr->colidx, 0, u, nb, uniq, rank);
            TRYC(cudaFuncSetAttribute(k_dedup_bitmap<32>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bm_smem));
            k_dedup_bitmap<32><<<(unsigned)W, kBmThreads, bm_smem, s>>>(M, K, nnz, csr->rowptr, csr->colidx, 0, u, nb,
                                                                       uniq, rank);
        }
        exclusive_scan_i64(nb, nb, W, tmp, s);
    } else {
        TRYC(cudaMemsetAsync(nb, 0, sizeof(int64_t), s));
    }
    TRYC(cudaGetLastError());
    TRYC(cudaMemcpyAsync(h.data(), nb, (W + 1) * sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    TRYC(cudaMemcpyAsync(&hflags, flags, sizeof(int), cudaMemcpyDeviceToHost, s));
    TRYC(cudaStreamSynchronize(s));
    if (hflags) {
        if (hflags & F_INVALID) { set_error("malformed rowptr"); rc = DTC_ERR_INVALID; }
        else if (hflags & F_RANGE) { set_error("column index out of [0, K)"); rc = DTC_ERR_RANGE; }
        else if (hflags & F_DUPLICATE) { set_error("duplicate column within a row"); rc = DTC_ERR_DUPLICATE; }
        else { set_error("columns not ascending within a row"); rc = DTC_ERR_UNSORTED; }
        goto done;
    }
    if (h[W] >= INT32_MAX / 8) { set_error("NumTCBlock too large"); rc = DTC_ERR_UNSUPPORTED; goto done; }
    rwo_out->assign((size_t)W + 1, 0);
    for (int64_t w = 0; w <= W; ++w) (*rwo_out)[(size_t)w] = (int32_t)h[(size_t)w];
done:
    cudaGetLastError();
    dfree(flags, s); dfree(u, s); dfree(nb, s); dfree(uniq, s); dfree(rank, s); dfree(tmp, s);
    cudaStreamSynchronize(s);
    return rc;
#undef TRY
#undef TRYC
}

}  // namespace dtc

using namespace dtc;

extern "C" int dtc_format_build_ex(const dtc_csr_t* csr, const dtc_build_opts_t* opts, void* stream,
                                   dtc_handle_t* out) {
    return format_build(csr, opts, (cudaStream_t)stream, out);
}

extern "C" int dtc_format_build(const dtc_csr_t* csr, void* stream, dtc_handle_t* out) {
    return format_build(csr, nullptr, (cudaStream_t)stream, out);
}

extern "C" int dtc_format_query(dtc_handle_t h, dtc_format_view_t* v) {
    if (!h || !v) { set_error("null handle or view"); return DTC_ERR_INVALID; }
    v->M = h->M; v->K = h->K; v->nnz = h->nnz; v->num_windows = h->W; v->num_tc_blocks = h->T;
    v->num_units = h->num_units; v->num_split_windows = h->num_split;
    v->dtype = h->dtype; v->unit_blocks = h->unit_blocks; v->window_rows = h->window_h;
    v->row_window_offset = h->rwo; v->tc_offset = h->tco; v->tc_local_id = h->lid;
    v->sparse_a_to_b = h->atob; v->tc_values = h->vals; v->units = (const int32_t*)h->units;
    return DTC_OK;
}

extern "C" int dtc_format_export(dtc_handle_t h, int32_t* rwo, int32_t* tco, uint8_t* lid, int32_t* atob,
                                 void* vals, int32_t* units) {
    if (!h) { set_error("null handle"); return DTC_ERR_INVALID; }
    DTC_CUDA(cudaDeviceSynchronize());
    if (rwo) DTC_CUDA(cudaMemcpy(rwo, h->rwo, (h->W + 1) * sizeof(int32_t), cudaMemcpyDeviceToHost));
    if (tco) DTC_CUDA(cudaMemcpy(tco, h->tco, (h->T + 1) * sizeof(int32_t), cudaMemcpyDeviceToHost));
    if (lid && h->nnz) DTC_CUDA(cudaMemcpy(lid, h->lid, h->nnz, cudaMemcpyDeviceToHost));
    if (atob && h->T) DTC_CUDA(cudaMemcpy(atob, h->atob, 8 * h->T * sizeof(int32_t), cudaMemcpyDeviceToHost));
    if (vals && h->nnz) DTC_CUDA(cudaMemcpy(vals, h->vals, h->nnz * elt_size(h->dtype), cudaMemcpyDeviceToHost));
    if (units && h->num_units) DTC_CUDA(cudaMemcpy(units, h->units, h->num_units * sizeof(Unit), cudaMemcpyDeviceToHost));
    return DTC_OK;
}

extern "C" void dtc_format_destroy(dtc_handle_t h) {
    if (!h) return;
    int prev = 0;
    cudaGetDevice(&prev);
    cudaSetDevice(h->device);
    cudaDeviceSynchronize();
    free_format(h, 0);
    cudaDeviceSynchronize();
    cudaSetDevice(prev);
    delete h;
}
