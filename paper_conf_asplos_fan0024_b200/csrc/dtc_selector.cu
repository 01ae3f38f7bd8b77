// dtc_selector.cu -- the simulation-based Selector as a diagnostic.
//
// PAPER.md:335-348 (§4.5.2, Eq. (1), Fig. 10): the makespan of the base kernel (one
// thread block per row window, length = the window's TC-block count) is simulated with
// the TB-scheduling model sm_idx = 2 (b mod 64) + (floor(b/64) mod 2) on 128 SMs and
// `occupancy` resident blocks per SM; the strict-balance makespan is
// NumTCBlocks / (SMs x occupancy); AR = base / balanced, and the balanced kernel is
// chosen when AR > 1.2.  Generalised to S SMs with 64 -> S/2 (reading C20/C23 in
// DESIGN.md): every block goes to SM eq1(b); on each SM the blocks take, in index order,
// the first freed of `occupancy` slots (the paper's "block 128 completes, block 768 is
// scheduled", which is SM 0 under Eq. (1)).
//
// On B200 the product always runs the F4 TC-block-balanced units (the balance is free of
// atomics there), so this is reported, not used to switch kernels.
#include <vector>

#include "dtc_internal.h"

using namespace dtc;

extern "C" int dtc_selector_ar(const int32_t* rwo, int64_t W, int32_t num_sms, int32_t occupancy,
                               double* makespan_base, double* makespan_balanced, double* ar) {
    if (!rwo || W < 0 || num_sms < 2 || (num_sms & 1) || occupancy < 1 || occupancy > 1024) {
        set_error("bad selector arguments (num_sms must be even and >= 2, occupancy 1..1024)");
        return DTC_ERR_INVALID;
    }
    const int64_t half = num_sms / 2;
    std::vector<int64_t> slot((size_t)num_sms * occupancy, 0);   // finish time of each resident slot
    for (int64_t b = 0; b < W; ++b) {
        const int64_t len = (int64_t)rwo[b + 1] - rwo[b];
        if (len < 0) { set_error("RowWindowOffset not monotone at %lld", (long long)b); return DTC_ERR_INVALID; }
        const int64_t sm = 2 * (b % half) + ((b / half) % 2);   // Eq. (1)
        int64_t* s = slot.data() + sm * occupancy;
        int j = 0;                                               // first-freed slot (lowest index on ties)
        for (int k = 1; k < occupancy; ++k)
            if (s[k] < s[j]) j = k;
        s[j] += len;
    }
    int64_t base = 0;
    for (int64_t t : slot) base = t > base ? t : base;
    const double T = (double)(W > 0 ? rwo[W] - rwo[0] : 0);
    const double bal = T / ((double)num_sms * occupancy);
    if (makespan_base) *makespan_base = (double)base;
    if (makespan_balanced) *makespan_balanced = bal;
    if (ar) *ar = bal > 0 ? (double)base / bal : 1.0;
    return DTC_OK;
}

// ======================================================================= B200 Selector (planner)
// The paper's Selector simulates the thread-block schedule of its base kernel to
// decide whether balancing pays (AR > 1.2).  On B200 the product always runs TC-block-balanced F4
// units, so the decision left is HOW to cut them: the unit size U (CTA length in TC blocks), the
// guided tail, and -- through U -- how many pieces long windows split into.  The retargeted
// Selector simulates OUR launch the paper's way: the units the builder would emit for a candidate
// (exactly: the F4 rules of dtc_sched.h), dispatched in unit order onto num_sms x occupancy
// resident-CTA slots (the measured occupancy of the kernel that will run; each unit takes the
// earliest-free slot, ties to the lowest slot -- in-order hardware CTA dispatch), each unit
// holding its slot for cta_ns + block_ns * nb, and the last piece of a split window additionally
// for the fixup chain fixup_ns * (G + ceil(np / G)) (G = fixup_group(np); the pieces of a window
// are consecutive and equal-sized, so its last piece is the one that finishes last).  The plan
// with the smallest simulated makespan wins (ties: larger U).
#include <algorithm>
#include <functional>
#include <queue>
#include <thread>

#include "dtc_sched.h"

namespace dtc {

// The unit list dtc_format_build emits for (U, tail) -- host version of k_units_count / fill / fix and
// the default split-pieces-first order.  Only {nb, split window id, piece, npieces} matter here.
struct SimUnit {
    int32_t nb, np, piece;
};

static void plan_units(const int32_t* rwo, int64_t W, int U, int64_t tail, std::vector<SimUnit>& split_units,
                       std::vector<SimUnit>& whole_units) {
    const int64_t T = W > 0 ? (int64_t)rwo[W] - rwo[0] : 0;
    const Guide gd = make_guide(T, U, tail);
    split_units.clear();
    whole_units.clear();
    int64_t cur_nb = -1;   // blocks of the open whole-window unit
    for (int64_t w = 0; w < W; ++w) {
        const int64_t nb = (int64_t)rwo[w + 1] - rwo[w];
        const int64_t Uw = gd.size_at(rwo[w]);
        if (nb > Uw) {
            const int64_t c = split_pieces(nb, Uw);
            for (int64_t p = 0; p < c; ++p) {
                const int64_t b0 = p * nb / c, b1 = (p + 1) * nb / c;
                split_units.push_back({(int32_t)(b1 - b0), (int32_t)c, (int32_t)p});
            }
            if (cur_nb >= 0) { whole_units.push_back({(int32_t)cur_nb, 1, 0}); cur_nb = -1; }
            continue;
        }
        bool starts = (w == 0) || cur_nb < 0;
        if (!starts) {
            const int64_t pnb = (int64_t)rwo[w] - rwo[w - 1];
            starts = (pnb > gd.size_at(rwo[w - 1])) || (gd.chunk(rwo[w]) != gd.chunk(rwo[w - 1]));
        }
        if (starts) {
            if (cur_nb >= 0) whole_units.push_back({(int32_t)cur_nb, 1, 0});
            cur_nb = 0;
        }
        cur_nb += nb;
    }
    if (cur_nb >= 0) whole_units.push_back({(int32_t)cur_nb, 1, 0});
}

static double simulate_units(const SimUnit* u, int64_t n, const dtc_sched_model_t& m) {
    const int64_t slots = (int64_t)m.num_sms * m.occupancy;
    // min-heap of (free time, slot): the earliest-free slot takes the next unit, lowest slot on ties
    using E = std::pair<double, int64_t>;
    std::priority_queue<E, std::vector<E>, std::greater<E>> q;
    for (int64_t k = 0; k < slots; ++k) q.push({0.0, k});
    double makespan = 0.0;
    for (int64_t i = 0; i < n; ++i) {
        E e = q.top();
        q.pop();
        double t = m.cta_ns + m.block_ns * u[i].nb;
        if (u[i].np > 1 && u[i].piece == u[i].np - 1) {
            const int G = fixup_group(u[i].np);
            t += m.fixup_ns * (G + (u[i].np + G - 1) / G);
        }
        e.first += t;
        makespan = std::max(makespan, e.first);
        q.push(e);
    }
    return makespan;
}

static bool model_ok(const dtc_sched_model_t* m) {
    return m && m->num_sms >= 1 && m->occupancy >= 1 && m->occupancy <= 1024 && m->cta_ns >= 0 && m->block_ns > 0 &&
           m->fixup_ns >= 0;
}

int selector_plan(const int32_t* rwo, int64_t W, const dtc_sched_model_t& m, const int32_t* cand, int ncand,
                  int guided_opt, dtc_plan_t* plans, dtc_plan_t* best) {
    static const int32_t kDefault[] = {16, 24, 32, 48, 64, 96, 128, 192, 256, 384, 512};
    if (!cand || ncand <= 0) {
        cand = kDefault;
        ncand = (int)(sizeof(kDefault) / sizeof(kDefault[0]));
    }
    for (int64_t w = 0; w < W; ++w)
        if (rwo[w + 1] < rwo[w]) { set_error("RowWindowOffset not monotone at %lld", (long long)w); return DTC_ERR_INVALID; }
    for (int i = 0; i < ncand; ++i)
        if (cand[i] < 8) { set_error("candidate unit size %d < 8", cand[i]); return DTC_ERR_INVALID; }
    const int64_t T = W > 0 ? (int64_t)rwo[W] - rwo[0] : 0;
    const int64_t slots = (int64_t)m.num_sms * m.occupancy;
    // plan k: candidate k / 2, guided tail (k odd) over ~4 U blocks per slot-ful of SMs
    const int nplans = 2 * ncand;
    std::vector<dtc_plan_t> out((size_t)nplans);
    auto run = [&](int k) {
        const int U = cand[k / 2];
        const int g = k & 1;
        dtc_plan_t& p = out[(size_t)k];
        p.unit_blocks = U;
        p.guided = g;
        if ((guided_opt > 0 && !g) || (guided_opt < 0 && g)) {   // excluded by the caller's choice
            p.num_units = -1;
            p.makespan_ns = -1.0;
            return;
        }
        std::vector<SimUnit> su, wu;
        plan_units(rwo, W, U, g ? (int64_t)m.num_sms * 4 * U : 0, su, wu);
        su.insert(su.end(), wu.begin(), wu.end());   // split pieces first (the builder's default order)
        p.num_units = (int64_t)su.size();
        p.makespan_ns = simulate_units(su.data(), (int64_t)su.size(), m);
    };
    const unsigned nt = std::max(1u, std::min<unsigned>(std::thread::hardware_concurrency(), (unsigned)nplans));
    if (nt <= 1 || T < 100000) {
        for (int k = 0; k < nplans; ++k) run(k);
    } else {
        std::vector<std::thread> th;
        for (unsigned t = 0; t < nt; ++t)
            th.emplace_back([&, t]() {
                for (int k = (int)t; k < nplans; k += (int)nt) run(k);
            });
        for (auto& x : th) x.join();
    }
    (void)slots;
    int bi = -1;
    for (int k = 0; k < nplans; ++k) {
        if (out[(size_t)k].makespan_ns < 0) continue;
        if (bi < 0 || out[(size_t)k].makespan_ns < out[(size_t)bi].makespan_ns ||
            (out[(size_t)k].makespan_ns == out[(size_t)bi].makespan_ns &&
             out[(size_t)k].unit_blocks > out[(size_t)bi].unit_blocks))
            bi = k;
    }
    if (plans) std::copy(out.begin(), out.end(), plans);
    if (best) {
        if (bi >= 0) *best = out[(size_t)bi];
        else *best = dtc_plan_t{cand[0], 0, 0, 0.0};
    }
    return DTC_OK;
}

}  // namespace dtc

extern "C" int dtc_selector_plan(const int32_t* rwo, int64_t W, const dtc_sched_model_t* m, const int32_t* cand_u,
                                 int32_t ncand, int32_t guided, dtc_plan_t* plans, dtc_plan_t* best) {
    if (!rwo || W < 0 || !model_ok(m)) { set_error("bad selector_plan arguments"); return DTC_ERR_INVALID; }
    return selector_plan(rwo, W, *m, cand_u, ncand, guided, plans, best);
}

extern "C" int dtc_selector_simulate(const int32_t* units, int64_t nu, const dtc_sched_model_t* m, double* makespan_ns) {
    if ((!units && nu > 0) || nu < 0 || !model_ok(m) || !makespan_ns) {
        set_error("bad selector_simulate arguments");
        return DTC_ERR_INVALID;
    }
    std::vector<SimUnit> su((size_t)nu);
    for (int64_t i = 0; i < nu; ++i) {
        const int32_t* r = units + 8 * i;   // {wb, we, bb, be, split_id, piece, npieces, slot_base}
        if (r[3] < r[2] || r[6] < 1 || r[5] < 0 || r[5] >= r[6]) { set_error("bad unit record %lld", (long long)i); return DTC_ERR_INVALID; }
        su[(size_t)i] = {r[3] - r[2], r[4] >= 0 ? r[6] : 1, r[4] >= 0 ? r[5] : 0};
    }
    *makespan_ns = simulate_units(su.data(), nu, *m);
    return DTC_OK;
}

namespace dtc {

// Default B200 schedule model for dtype and N on the current device (constants measured in round 1,
// DESIGN.md §5): a CTA holds its slot ~2.5 us beyond its blocks (start -> first B data ~2.3 us in
// the CTA trace, profiles/r01_cta_trace.txt, plus the epilogue); the gather of a TC block moves
// 8 rows x the CTA's columns through the SM's TMA unit, whose gather4 throughput is ~62.8 B/ns per SM
// (9.3 TB/s over 148 SMs, profiles/r01_gather_microbench.txt) and is shared by the SM's `occupancy`
// resident CTAs; one dependent partial load of a split fixup ~1 us.
constexpr double kCtaNs = 2500.0;
constexpr double kGatherBytesPerNsPerSm = 9296.0 / 148.0;
constexpr double kFixupNs = 1000.0;

int sched_model(int dtype, int64_t N, dtc_sched_model_t* m, int window_h) {
    if (N < 1) N = 1;
    const int occ = pad_occupancy(dtype, N, window_h);
    if (occ < 1) { set_error("cannot query the SpMM kernel occupancy"); return DTC_ERR_CUDA; }
    const PadGeometry g = pad_geometry(dtype, N, 0);
    const int64_t cols = std::min<int64_t>(N, window_h == 16 ? g.cta_cols : g.cta_cols / g.slices);
    m->num_sms = num_sms();
    m->occupancy = occ;
    m->cta_ns = kCtaNs;
    m->block_ns = occ * 8.0 * (double)cols * elt_size(dtype) / kGatherBytesPerNsPerSm;
    m->fixup_ns = kFixupNs;
    return DTC_OK;
}

}  // namespace dtc

extern "C" int dtc_sched_model(int32_t dtype, int64_t N, dtc_sched_model_t* m) {
    if (!m || (dtype != DTC_TF32 && dtype != DTC_FP16)) { set_error("bad sched_model arguments"); return DTC_ERR_INVALID; }
    int n = 0;
    if (cudaGetDeviceCount(&n) != cudaSuccess || n == 0) { cudaGetLastError(); set_error("no CUDA device"); return DTC_ERR_CUDA; }
    return sched_model(dtype, N, m, 16);
}
