// dtc_tca.cu -- TCU-Cache-Aware (TCA) row reordering, §4.3, Alg. 1
// (optional host preprocessing; north_star: "an optional host preprocessing step").
//
// Hierarchy I (TCU-aware, Alg. 1 l.1-14): candidate row pairs from MinHash-LSH over
// the rows' column sets, exact Jaccard, a priority queue (most similar first), and
// cluster merging while clusters are below BLOCK_HEIGHT = 16 rows; a cluster that
// reaches 16 rows leaves the pool.
// Hierarchy II (cache-aware, l.15-28): the same over row clusters (deduplicated
// column sets) with the limit SM_NUM clusters per cluster-of-clusters.
// Reid (l.29): rows ordered by cluster of clusters, then row cluster, then row.
//
// Readings where Alg. 1 is silent (T1-T8): MinHash with 16 hash
// functions h_m(c) = mix64(c, m); LSH with 8 bands of 2; within a band bucket
// (sorted by (key, index)) each member pairs with its next 8 members; exact Jaccard
// with ties broken by (i, j) ascending and exact rational comparison; pairs whose
// clusters coincide or already left the pool are skipped; leftover pool clusters
// join the next hierarchy / the final order; clusters ordered by smallest row id.
// An independent step-by-step Python transcription under tests' control implements
// the same steps; tests compare the permutations exactly.
#include <algorithm>
#include <cstdint>
#include <cstring>
#include <numeric>
#include <thread>
#include <vector>

#include "dtc_internal.h"

namespace dtc {
namespace tca {

constexpr int kHashes = 16;      // T1
constexpr int kBands = 8;        // T2: 8 bands x 2 rows
constexpr int kRowsPerBand = kHashes / kBands;
constexpr int kNeighbours = 8;   // T3: pairs per bucket member

static inline uint64_t mix64(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}
static inline uint32_t hash_m(uint32_t c, int m) {
    return (uint32_t)(mix64(((uint64_t)c << 8) ^ (uint64_t)(m + 1) * 0xD1B54A32D192ED03ull) >> 32);
}

struct Pair {
    int32_t i, j;        // i < j
    int64_t inter, uni;  // Jaccard = inter / uni
};

// "a more similar than b": Jaccard descending (exact), then (i, j) ascending (T4)
static inline bool before(const Pair& a, const Pair& b) {
    const __int128 l = (__int128)a.inter * b.uni, r = (__int128)b.inter * a.uni;
    if (l != r) return l > r;
    if (a.i != b.i) return a.i < b.i;
    return a.j < b.j;
}

static int64_t inter_size(const int32_t* a, int64_t na, const int32_t* b, int64_t nb) {
    int64_t x = 0, y = 0, k = 0;
    while (x < na && y < nb) {
        if (a[x] < b[y]) ++x;
        else if (a[x] > b[y]) ++y;
        else { ++k; ++x; ++y; }
    }
    return k;
}

// MinhashLSH over n sorted sets (offsets/items); returns candidate pairs with J > 0, sorted.
static std::vector<Pair> minhash_lsh(int64_t n, const std::vector<int64_t>& off, const std::vector<int32_t>& items) {
    std::vector<uint32_t> sig((size_t)n * kHashes, 0xFFFFFFFFu);
    for (int64_t i = 0; i < n; ++i)
        for (int64_t p = off[i]; p < off[i + 1]; ++p)
            for (int m = 0; m < kHashes; ++m) {
                const uint32_t h = hash_m((uint32_t)items[p], m);
                uint32_t& s = sig[(size_t)i * kHashes + m];
                if (h < s) s = h;
            }
    std::vector<std::pair<uint64_t, int32_t>> bucket;
    bucket.reserve((size_t)n);
    std::vector<std::pair<int32_t, int32_t>> cand;
    for (int band = 0; band < kBands; ++band) {
        bucket.clear();
        for (int64_t i = 0; i < n; ++i) {
            if (off[i + 1] == off[i]) continue;   // empty sets never pair
            uint64_t key = (uint64_t)band * 0x9E3779B97F4A7C15ull;
            for (int r = 0; r < kRowsPerBand; ++r) key = mix64(key ^ sig[(size_t)i * kHashes + band * kRowsPerBand + r]);
            bucket.push_back({key, (int32_t)i});
        }
        std::sort(bucket.begin(), bucket.end());
        for (size_t a = 0; a < bucket.size(); ++a)
            for (size_t b = a + 1; b < bucket.size() && b <= a + kNeighbours && bucket[b].first == bucket[a].first; ++b)
                cand.push_back({bucket[a].second, bucket[b].second});
    }
    std::sort(cand.begin(), cand.end());
    cand.erase(std::unique(cand.begin(), cand.end()), cand.end());
    std::vector<Pair> pairs;
    pairs.reserve(cand.size());
    for (auto& c : cand) {
        const int32_t i = c.first, j = c.second;
        const int64_t ni = off[i + 1] - off[i], nj = off[j + 1] - off[j];
        const int64_t in = inter_size(&items[off[i]], ni, &items[off[j]], nj);
        if (in > 0) pairs.push_back({i, j, in, ni + nj - in});
    }
    std::sort(pairs.begin(), pairs.end(), before);
    return pairs;
}

// Alg. 1 merge loop: clusters of the n items, merged along `pairs` in queue order
// while both are in the pool; a merged cluster whose size (in items) reaches `limit`
// leaves the pool.  Returns the clusters, each sorted ascending.
static std::vector<std::vector<int32_t>> merge_clusters(int64_t n, const std::vector<Pair>& pairs, int64_t limit) {
    std::vector<int32_t> owner((size_t)n);
    std::vector<std::vector<int32_t>> members((size_t)n);
    std::vector<char> in_pool((size_t)n, 1);
    for (int64_t i = 0; i < n; ++i) {
        owner[i] = (int32_t)i;
        members[i] = {(int32_t)i};
    }
    for (const Pair& p : pairs) {
        const int32_t ci = owner[p.i], cj = owner[p.j];          // FindCluster
        if (ci == cj || !in_pool[ci] || !in_pool[cj]) continue;  // T5
        const int32_t keep = std::min(ci, cj), drop = std::max(ci, cj);
        for (int32_t x : members[drop]) owner[x] = keep;         // Merge
        members[keep].insert(members[keep].end(), members[drop].begin(), members[drop].end());
        members[drop].clear();
        in_pool[drop] = 0;
        if ((int64_t)members[keep].size() >= limit) in_pool[keep] = 0;   // -> RC_set / CC_set
    }
    std::vector<std::vector<int32_t>> out;
    for (int64_t c = 0; c < n; ++c)
        if (!members[c].empty()) {
            std::sort(members[c].begin(), members[c].end());
            out.push_back(std::move(members[c]));
        }
    return out;   // ordered by smallest member (T7)
}

}  // namespace tca
}  // namespace dtc

using namespace dtc;

extern "C" int dtc_tca_reorder(int64_t M, int64_t K, const int32_t* rowptr, const int32_t* colidx, int32_t sm_num,
                               int32_t* perm) {
    if (M < 0 || K < 0 || !perm || (M > 0 && (!rowptr || !colidx)) || sm_num < 1) {
        set_error("bad arguments to dtc_tca_reorder");
        return DTC_ERR_INVALID;
    }
    try {
        // Hierarchy I over rows
        std::vector<int64_t> off(M + 1);
        for (int64_t i = 0; i <= M; ++i) off[i] = rowptr[i];
        std::vector<int32_t> items(colidx, colidx + (M > 0 ? rowptr[M] : 0));
        auto rpairs = tca::minhash_lsh(M, off, items);
        auto rc = tca::merge_clusters(M, rpairs, kWindow);
        // Hierarchy II over row clusters: deduplicated column set of each cluster
        const int64_t nc = (int64_t)rc.size();
        std::vector<int64_t> coff(nc + 1, 0);
        std::vector<int32_t> citems;
        for (int64_t c = 0; c < nc; ++c) {
            std::vector<int32_t> u;
            for (int32_t r : rc[c]) u.insert(u.end(), colidx + rowptr[r], colidx + rowptr[r + 1]);
            std::sort(u.begin(), u.end());
            u.erase(std::unique(u.begin(), u.end()), u.end());
            citems.insert(citems.end(), u.begin(), u.end());
            coff[c + 1] = (int64_t)citems.size();
        }
        auto cpairs = tca::minhash_lsh(nc, coff, citems);
        auto cc = tca::merge_clusters(nc, cpairs, sm_num);
        // Reid: clusters of clusters by smallest row, row clusters by smallest row, rows ascending (T7)
        std::vector<std::pair<int32_t, int32_t>> cc_order;   // (smallest row, index)
        for (size_t k = 0; k < cc.size(); ++k) {
            int32_t mn = INT32_MAX;
            for (int32_t c : cc[k]) mn = std::min(mn, rc[c].front());
            cc_order.push_back({mn, (int32_t)k});
        }
        std::sort(cc_order.begin(), cc_order.end());
        int64_t pos = 0;
        for (auto& ko : cc_order) {
            std::vector<std::pair<int32_t, int32_t>> rcs;
            for (int32_t c : cc[ko.second]) rcs.push_back({rc[c].front(), c});
            std::sort(rcs.begin(), rcs.end());
            for (auto& x : rcs)
                for (int32_t r : rc[x.second]) perm[pos++] = r;
        }
        if (pos != M) { set_error("internal: permutation incomplete"); return DTC_ERR_INVALID; }
    } catch (const std::bad_alloc&) {
        set_error("host OOM in dtc_tca_reorder");
        return DTC_ERR_OOM;
    }
    return DTC_OK;
}

// NumTCBlock of the matrix with rows in `perm` order (NULL = identity): sum over 16-row windows of
// ceil(|unique columns| / 8), host threads over windows.
static int64_t count_tc_blocks(int64_t M, const int32_t* rowptr, const int32_t* colidx, const int32_t* perm) {
    const int64_t W = (M + kWindow - 1) / kWindow;
    const unsigned nt = std::max(1u, std::min(16u, std::thread::hardware_concurrency()));
    std::vector<int64_t> part(nt, 0);
    std::vector<std::thread> th;
    for (unsigned t = 0; t < nt; ++t)
        th.emplace_back([&, t]() {
            std::vector<int32_t> u;
            int64_t acc = 0;
            for (int64_t w = t; w < W; w += nt) {
                u.clear();
                for (int64_t r = w * kWindow; r < std::min(M, (w + 1) * kWindow); ++r) {
                    const int64_t row = perm ? perm[r] : r;
                    u.insert(u.end(), colidx + rowptr[row], colidx + rowptr[row + 1]);
                }
                std::sort(u.begin(), u.end());
                const int64_t nu = std::unique(u.begin(), u.end()) - u.begin();
                acc += (nu + kTcw - 1) / kTcw;
            }
            part[t] = acc;
        });
    for (auto& x : th) x.join();
    int64_t T = 0;
    for (int64_t v : part) T += v;
    return T;
}

extern "C" int dtc_tca_reorder_checked(int64_t M, int64_t K, const int32_t* rowptr, const int32_t* colidx,
                                       int32_t sm_num, int32_t* perm, int64_t* T_identity, int64_t* T_reordered,
                                       int32_t* applied) {
    const int rc = dtc_tca_reorder(M, K, rowptr, colidx, sm_num, perm);
    if (rc != DTC_OK) return rc;
    try {
        const int64_t t0 = count_tc_blocks(M, rowptr, colidx, nullptr);
        const int64_t t1 = count_tc_blocks(M, rowptr, colidx, perm);
        const bool use = t1 < t0;
        if (!use)
            for (int64_t i = 0; i < M; ++i) perm[i] = (int32_t)i;
        if (T_identity) *T_identity = t0;
        if (T_reordered) *T_reordered = t1;
        if (applied) *applied = use ? 1 : 0;
    } catch (const std::exception&) {
        set_error("host failure in dtc_tca_reorder_checked");
        return DTC_ERR_OOM;
    }
    return DTC_OK;
}
