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
