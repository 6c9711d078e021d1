// shard_plan.cpp -- host-only shard planner (include/ffm.h ffm_shard_plan).
//
// SITE_LPT: whole call sites are bin-packed over the ranks by payload bytes, largest
// first onto the least-loaded rank (LPT).  Every re-upload of a site stays on one rank,
// so the dominant duplicate pattern -- the same data re-sent from the same call site
// every loop iteration -- never crosses a shard; only
// cross-site shared content does.
// CONTIGUOUS: contiguous gid ranges with ~equal bytes (the stress case).
#include <stdint.h>

#include <algorithm>
#include <numeric>
#include <vector>

#include "../../include/ffm.h"

extern "C" int ffm_shard_plan(uint64_t n, const uint32_t* sites, const uint64_t* sizes, uint32_t n_sites,
                              int32_t world, int policy, int32_t* rank_out) {
    if (world < 1 || (n && (!sites || !sizes || !rank_out)) || n_sites == 0) return FFM_E_INVAL;
    if (policy != FFM_SHARD_SITE_LPT && policy != FFM_SHARD_CONTIGUOUS) return FFM_E_INVAL;
    for (uint64_t i = 0; i < n; ++i)
        if (sites[i] >= n_sites) return FFM_E_RANGE;
    try {
        if (policy == FFM_SHARD_CONTIGUOUS) {
            long double total = 0;
            for (uint64_t i = 0; i < n; ++i) total += (long double)sizes[i] + 1;   // +1: empty records count
            long double acc = 0;
            for (uint64_t i = 0; i < n; ++i) {
                long double mid = acc + ((long double)sizes[i] + 1) / 2;
                int r = total > 0 ? (int)(mid * world / total) : 0;
                rank_out[i] = std::min<int>(std::max(r, 0), world - 1);
                acc += (long double)sizes[i] + 1;
            }
            return FFM_OK;
        }
        std::vector<uint64_t> bytes(n_sites, 0);
        for (uint64_t i = 0; i < n; ++i) bytes[sites[i]] += sizes[i] + 1;
        std::vector<uint32_t> order(n_sites);
        std::iota(order.begin(), order.end(), 0u);
        std::stable_sort(order.begin(), order.end(), [&](uint32_t a, uint32_t b) { return bytes[a] > bytes[b]; });
        std::vector<uint64_t> load(world, 0);
        std::vector<int32_t> site_rank(n_sites, 0);
        for (uint32_t s : order) {
            if (!bytes[s]) break;
            int best = 0;
            for (int r = 1; r < world; ++r)
                if (load[r] < load[best]) best = r;
            site_rank[s] = best;
            load[best] += bytes[s];
        }
        for (uint64_t i = 0; i < n; ++i) rank_out[i] = site_rank[sites[i]];
    } catch (...) {
        return FFM_E_NOMEM;
    }
    return FFM_OK;
}
