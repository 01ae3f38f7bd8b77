// dtc_sched.h -- the F4 work-unit rules shared by the builder (dtc_format.cu, on the GPU), the
// kernel's split fixup (dtc_spmm.cu) and the B200 Selector's host simulation (dtc_selector.cu),
// so the Selector plans exactly the units the builder would emit.
#pragma once
#include <cmath>
#include <cstdint>

namespace dtc {

// Work units: consecutive windows whose first TC block falls in the same chunk form
// one unit; a window with more blocks than its chunk size is split into near-equal pieces (each
// its own unit, deterministic fixup).  Chunk sizes are "guided": U blocks, then U/2 over the last
// ~half wave of blocks, so the CTAs dispatched last are short and the tail of the grid is even.
struct Guide {
    int64_t x[5];     // segment starts (x[4] = T)
    int64_t sz[4];    // chunk size per segment
    int64_t off[4];   // chunk-id offset per segment
    __host__ __device__ int seg(int64_t v) const {
        int k = 0;
        while (k < 3 && v >= x[k + 1]) ++k;
        return k;
    }
    __host__ __device__ int64_t chunk(int64_t v) const {
        const int k = seg(v);
        return off[k] + (v - x[k]) / sz[k];
    }
    __host__ __device__ int64_t size_at(int64_t v) const { return sz[seg(v)]; }
};

inline Guide make_guide(int64_t T, int U, int64_t tail_span) {
    Guide g;
    int64_t A = tail_span > T ? T : tail_span;
    g.x[0] = 0;
    g.x[1] = T - A;
    g.x[2] = T - A / 2;
    g.x[3] = T - A / 4;
    g.x[4] = T;
    // sizes U, then U/2 for the rest of the tail (smaller units lose more to per-unit
    // startup than they win at the end of the grid -- measured)
    for (int k = 0; k < 4; ++k) {
        const int64_t sz = k == 0 ? U : U / 2;
        g.sz[k] = sz < 8 ? 8 : sz;
    }
    g.off[0] = 0;
    for (int k = 1; k < 4; ++k) g.off[k] = g.off[k - 1] + (g.x[k] - g.x[k - 1] + g.sz[k - 1] - 1) / g.sz[k - 1];
    return g;
}

// Pieces of a split window (nb > U blocks): at least U blocks each, and at most ~sqrt(nb/2) of them.
// A piece costs ~nb/np block times (~0.5 us each) and the last arriver's fixup chains ~2 sqrt(np)
// dependent partial loads (~1 us each), so the window's critical path is smallest near
// np = sqrt(nb/2) (c2's hub windows: ~1,600 blocks -> 29 pieces instead of 100 at U = 16).
__host__ __device__ inline int64_t split_pieces(int64_t nb, int64_t U) {
    const int64_t byU = (nb + U - 1) / U;
    int64_t r = (int64_t)sqrt((double)nb * 0.5);
    if (r < 1) r = 1;
    while (2 * r * r < nb) ++r;   // ceil(sqrt(nb/2))
    while (r > 1 && 2 * (r - 1) * (r - 1) >= nb) --r;
    return byU < r ? byU : r;
}

// Split fixup group size: a window split into np pieces forms groups of G = ceil(sqrt(np))
// consecutive pieces (one group when np <= 4); the dependent chain is G + np/G partial loads.
__host__ __device__ inline int fixup_group(int np) {
    if (np <= 4) return np;
    int g = 1;
    while (g * g < np) ++g;
    return g;
}

}  // namespace dtc
