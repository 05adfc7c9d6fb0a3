// host_util.cpp — host-only parts of the C-ABI (no CUDA calls here):
// status strings, default options, the nnz-balanced partitioner, halo ghost
// lists, the performance-history table and its selection policy.
//
// Paper anchors (PAPER.md byte offsets):
//   partitioning of one call into sub-tasks, concatenated results: §IV-F P@27330–28000
//   history-based dynamic composition: §III P@10254–10489, default P@10778
//   context instance = tuple of context-property values: §III P@9781
//   "average case execution time" as the selection metric: §II P@4425
#include "pepp_internal.h"

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <unordered_map>
#include <string>
#include <vector>

namespace {
thread_local char g_last_error[512] = "";
}

void pepp::set_last_error(const char* msg, const char* expr, int line) {
    std::snprintf(g_last_error, sizeof(g_last_error), "%s (%s, plan.cu:%d)", msg ? msg : "?", expr ? expr : "?", line);
}

extern "C" PEPP_API const char* pepp_last_error(void) { return g_last_error; }

extern "C" PEPP_API const char* pepp_status_str(pepp_status_t s) {
    switch (s) {
    case PEPP_OK: return "PEPP_OK";
    case PEPP_E_INVALID: return "PEPP_E_INVALID: invalid argument or malformed CSR";
    case PEPP_E_CUDA: return "PEPP_E_CUDA: CUDA runtime error";
    case PEPP_E_NCCL: return "PEPP_E_NCCL: NCCL unavailable or failed";
    case PEPP_E_NOMEM: return "PEPP_E_NOMEM: out of memory";
    case PEPP_E_UNSUPPORTED: return "PEPP_E_UNSUPPORTED: valid input not supported";
    case PEPP_E_STATE: return "PEPP_E_STATE: call invalid in the current state";
    }
    return "PEPP_E_UNKNOWN";
}

extern "C" PEPP_API int32_t pepp_abi_version(void) { return PEPP_ABI_VERSION; }

extern "C" PEPP_API void pepp_spmv_opts_default(pepp_spmv_opts_t* o) {
    if (!o) return;
    std::memset(o, 0, sizeof(*o));
    o->variant_mask = 0;
    o->use_history = 1;
    o->validate = 1;
    o->sell_sigma = 0;
    o->device = -1;
    o->min_samples = 3;
    o->sample_period = 8;
    o->nranks = 1;
    o->rank = 0;
    o->row_bounds = nullptr;
    o->nccl_comm = nullptr;
    o->nccl_unique_id = nullptr;
    o->exchange = PEPP_X_AUTO;
    o->history_path = nullptr;
    o->prune = 1;
    o->overlap = 1;
    o->compress_values = 1;
    o->dist_select = 1;
    // the composition tool's global switches (§IV: disableImpls P@16687,
    // useHistoryModels "per component or global" P@28058) as environment
    // defaults: they set the defaults only — options a caller sets after
    // this call (the per-component form) win
    if (const char* v = std::getenv("PEPP_VARIANT")) {
        uint32_t m = 0;
        std::string list(v);
        size_t i = 0;
        while (i <= list.size()) {
            size_t j = list.find(',', i);
            if (j == std::string::npos) j = list.size();
            const std::string t = list.substr(i, j - i);
            if (t == "csr_vector") m |= 1u << PEPP_V_CSR_VECTOR;
            else if (t == "merge_path") m |= 1u << PEPP_V_MERGE_PATH;
            else if (t == "sell") m |= 1u << PEPP_V_SELL;
            else if (t == "csr_stream") m |= 1u << PEPP_V_CSR_STREAM;
            else if (t == "panel") m |= 1u << PEPP_V_PANEL;
            i = j + 1;
        }
        o->variant_mask = m;   // unknown names only: 0 = every variant
    }
    if (const char* v = std::getenv("PEPP_USE_HISTORY")) o->use_history = std::atoi(v) != 0;
    if (const char* v = std::getenv("PEPP_HISTORY_PATH")) if (*v) o->history_path = v;
}

// ---------------------------------------------------------------- partition
extern "C" PEPP_API pepp_status_t pepp_partition_rows(const int64_t* row_ptr, int64_t nrows, int64_t first,
                                                     int32_t nparts, int64_t* bounds) {
    if (!row_ptr || !bounds || nparts < 1 || nrows < 0) return PEPP_E_INVALID;
    const int64_t nnz = row_ptr[nrows] - first;
    if (nnz < 0 || row_ptr[0] != first) return PEPP_E_INVALID;
    bounds[0] = 0;
    for (int32_t p = 1; p < nparts; ++p) {
        // ceil(p*nnz/nparts), computed in 128-bit to be safe for huge nnz
        const __int128 num = (__int128)p * nnz + (nparts - 1);
        const int64_t target = (int64_t)(num / nparts);
        // smallest r with row_ptr[r] - first >= target (row_ptr non-decreasing)
        const int64_t* it = std::lower_bound(row_ptr, row_ptr + nrows + 1, target + first);
        bounds[p] = (int64_t)(it - row_ptr);
        if (bounds[p] < bounds[p - 1]) bounds[p] = bounds[p - 1];
    }
    bounds[nparts] = nrows;
    return PEPP_OK;
}

// ---------------------------------------------------------------- halo
extern "C" PEPP_API pepp_status_t pepp_halo_ghosts(const int32_t* col_idx, int64_t nnz, int32_t nranks, int32_t rank,
                                                  const int64_t* row_bounds, int64_t* counts, int32_t* ghosts,
                                                  int64_t cap, int64_t* total) {
    if ((!col_idx && nnz > 0) || nranks < 1 || rank < 0 || rank >= nranks || !row_bounds || !counts || !total)
        return PEPP_E_INVALID;
    std::vector<int32_t> g;
    pepp::halo_ghost_list(col_idx, nnz, row_bounds[rank], row_bounds[rank + 1], g);
    for (int32_t q = 0; q < nranks; ++q) counts[q] = 0;
    for (int32_t c : g) {
        // owner: largest q with row_bounds[q] <= c
        const int64_t* it = std::upper_bound(row_bounds, row_bounds + nranks + 1, (int64_t)c);
        int32_t q = (int32_t)(it - row_bounds) - 1;
        if (q < 0 || q >= nranks) return PEPP_E_INVALID;   // column beyond the partitioned range
        counts[q] += 1;
    }
    *total = (int64_t)g.size();
    if (ghosts && (int64_t)g.size() <= cap) std::memcpy(ghosts, g.data(), g.size() * sizeof(int32_t));
    return PEPP_OK;
}

namespace pepp {

void halo_ghost_list(const int32_t* col, int64_t nnz, int64_t lo, int64_t hi, std::vector<int32_t>& out) {
    // mark-and-sweep over the column range would need O(ncols) memory; sort the
    // outside-own-range columns instead (O(ghost_refs log ghost_refs)).
    out.clear();
    for (int64_t k = 0; k < nnz; ++k) {
        const int64_t c = col[k];
        if (c < lo || c >= hi) out.push_back((int32_t)c);
    }
    std::sort(out.begin(), out.end());
    out.erase(std::unique(out.begin(), out.end()), out.end());
}

// ---------------------------------------------------------------- history
struct HistKey {
    uint64_t key;
    int32_t cand;
    bool operator==(const HistKey& o) const { return key == o.key && cand == o.cand; }
};
struct HistKeyHash {
    size_t operator()(const HistKey& k) const { return std::hash<uint64_t>()(k.key * 1315423911ULL + (uint64_t)k.cand); }
};

}  // namespace pepp

struct pepp_history {
    std::unordered_map<pepp::HistKey, pepp::Welford, pepp::HistKeyHash> table;
};

namespace pepp {

void Welford::add(double v) {
    count += 1;
    const double d = v - mean;
    mean += d / (double)count;
    m2 += d * (v - mean);
}

pepp_history* history_new() { return new (std::nothrow) pepp_history(); }
void history_free(pepp_history* h) { delete h; }

void history_add(pepp_history* h, uint64_t key, int32_t cand, double us) { h->table[{key, cand}].add(us); }

const Welford* history_get(const pepp_history* h, uint64_t key, int32_t cand) {
    auto it = h->table.find({key, cand});
    return it == h->table.end() ? nullptr : &it->second;
}

double history_best_mean(const pepp_history* h, uint64_t key, int32_t ncand, const uint8_t* eligible) {
    double best = -1.0;
    for (int32_t c = 0; c < ncand; ++c) {
        if (!eligible[c]) continue;
        const Welford* w = history_get(h, key, c);
        if (w && w->count > 0 && (best < 0 || w->mean < best)) best = w->mean;
    }
    return best;
}

bool history_abandoned(const Welford* w, double best_mean) {
    return w && w->count > 0 && best_mean > 0 && w->mean > kAbandonFactor * best_mean;
}

bool history_contender(const Welford* w, double best_mean) {
    return w && w->count > 0 && best_mean > 0 && w->mean <= kContendFactor * best_mean;
}

int32_t history_pick(const pepp_history* h, uint64_t key, int32_t ncand, const uint8_t* eligible,
                     int32_t min_samples, int32_t* calibrating, double* predicted_us) {
    const double best_mean = history_best_mean(h, key, ncand, eligible);
    // 1) calibration in rounds: round r gives every candidate its r-th sample
    //    (lowest index first), skipping candidates already ruled out; rounds
    //    past min_samples (refinement) only for the contenders, those within
    //    kContendFactor of the best mean, when there are at least two — where
    //    measurement noise can flip the choice (short calls: event times come
    //    in ~2 µs steps)
    int32_t ncontend = 0;
    for (int32_t c = 0; c < ncand; ++c) ncontend += eligible[c] && history_contender(history_get(h, key, c), best_mean);
    const int32_t rounds = ncontend >= 2 ? kRefineRounds * min_samples : min_samples;
    for (int32_t r = 1; r <= rounds; ++r) {
        for (int32_t c = 0; c < ncand; ++c) {
            if (!eligible[c]) continue;
            const Welford* w = history_get(h, key, c);
            if (r > min_samples && !history_contender(w, best_mean)) continue;
            if ((!w || w->count < r) && !history_abandoned(w, best_mean)) {
                *calibrating = 1;
                *predicted_us = w ? w->mean : 0.0;
                return c;
            }
        }
    }
    // 2) exploitation: argmin of the mean, ties within 1 % -> lower index (A10)
    int32_t best = -1;
    double best_t = 0.0;
    for (int32_t c = 0; c < ncand; ++c) {
        if (!eligible[c]) continue;
        const Welford* w = history_get(h, key, c);
        if (!w || w->count == 0) continue;
        const double t = w->mean;
        if (best < 0 || t < best_t * 0.99) { best = c; best_t = t; }
    }
    *calibrating = 0;
    *predicted_us = best_t;
    return best;
}

// Cold start (static composition from recorded runs, P@10069 / P@10489): the
// nearest context key (bucket distance; same tag and rank count) that has
// samples for some of the given candidate ids; their means become a prior.
bool history_prior(const pepp_history* h, uint64_t key, int32_t n, const int32_t* ids, double* prior,
                   uint64_t* from_key) {
    auto field = [](uint64_t k, int shift, uint64_t mask) { return (int64_t)((k >> shift) & mask); };
    auto dist = [&](uint64_t a, uint64_t b) -> int64_t {
        if ((a >> 27) != (b >> 27)) return -1;   // ranks + instance + tag must match
        return std::llabs(field(a, 0, 0x7f) - field(b, 0, 0x7f)) + std::llabs(field(a, 7, 0x7f) - field(b, 7, 0x7f)) +
               std::llabs(field(a, 14, 0x7f) - field(b, 14, 0x7f)) + std::llabs(field(a, 21, 0x3f) - field(b, 21, 0x3f));
    };
    int64_t best_d = -1;
    uint64_t best_k = 0;
    for (const auto& kv : h->table) {
        const uint64_t k = kv.first.key;
        if (k == key || kv.second.count == 0) continue;
        bool ours = false;
        for (int32_t c = 0; c < n && !ours; ++c) ours = ids[c] == kv.first.cand;
        if (!ours) continue;
        const int64_t d = dist(key, k);
        if (d < 0) continue;
        if (best_d < 0 || d < best_d || (d == best_d && k < best_k)) { best_d = d; best_k = k; }
    }
    if (best_d < 0) return false;
    for (int32_t c = 0; c < n; ++c) {
        const Welford* w = history_get(h, best_k, ids[c]);
        prior[c] = (w && w->count > 0) ? w->mean : -1.0;
    }
    if (from_key) *from_key = best_k;
    return true;
}

int32_t dist_argmin(int32_t nd, const double* agreed, const uint8_t* eligible) {
    // argmin of the agreed means, ties within 1 % -> lower index (reading A10)
    int32_t c = -1;
    double bt = 0.0;
    for (int32_t d = 0; d < nd; ++d) {
        if ((eligible && !eligible[d]) || !(agreed[d] > 0.0) || std::isinf(agreed[d])) continue;
        if (c < 0 || agreed[d] < bt * 0.99) { c = d; bt = agreed[d]; }
    }
    return c;
}

uint64_t context_key(int64_t nrows, int64_t ncols, int64_t nnz, double cv, int32_t nparts, int32_t instance) {
    // bucketed context instance: half-octave buckets of rows / cols / nnz,
    // quarter buckets of the row-length CV (capped), and the partition count.
    auto hb = [](int64_t v) -> uint64_t { return (uint64_t)std::floor(2.0 * std::log2((double)v + 1.0)); };
    uint64_t cvb = (uint64_t)std::min(63.0, std::floor(4.0 * std::max(0.0, cv)));
    uint64_t k = 0;
    k |= (hb(nrows) & 0x7f);
    k |= (hb(ncols) & 0x7f) << 7;
    k |= (hb(nnz) & 0x7f) << 14;
    k |= (cvb & 0x3f) << 21;
    k |= ((uint64_t)nparts & 0xffff) << 27;
    k |= ((uint64_t)instance & 0x1f) << 43;   // kernel instance: value type, value compression
    k |= (uint64_t)0x5EBBu << 48;   // tag: CSR SpMV
    return k;
}

}  // namespace pepp

extern "C" PEPP_API pepp_status_t pepp_history_create(pepp_history** out) {
    if (!out) return PEPP_E_INVALID;
    *out = pepp::history_new();
    return *out ? PEPP_OK : PEPP_E_NOMEM;
}

extern "C" PEPP_API pepp_status_t pepp_history_destroy(pepp_history* h) {
    pepp::history_free(h);
    return PEPP_OK;
}

extern "C" PEPP_API pepp_status_t pepp_history_record(pepp_history* h, uint64_t key, int32_t cand, double us) {
    if (!h || cand < 0 || !(us >= 0.0) || std::isinf(us)) return PEPP_E_INVALID;
    pepp::history_add(h, key, cand, us);
    return PEPP_OK;
}

extern "C" PEPP_API pepp_status_t pepp_history_stats(const pepp_history* h, uint64_t key, int32_t cand,
                                                    int64_t* count, double* mean_us, double* m2) {
    if (!h) return PEPP_E_INVALID;
    const pepp::Welford* w = pepp::history_get(h, key, cand);
    if (count) *count = w ? w->count : 0;
    if (mean_us) *mean_us = w ? w->mean : 0.0;
    if (m2) *m2 = w ? w->m2 : 0.0;
    return PEPP_OK;
}

extern "C" PEPP_API pepp_status_t pepp_history_select(const pepp_history* h, uint64_t key, int32_t ncand,
                                                     const uint8_t* eligible, int32_t min_samples,
                                                     int32_t* cand, int32_t* calibrating, double* predicted_us) {
    if (!h || !eligible || !cand || !calibrating || !predicted_us || ncand <= 0) return PEPP_E_INVALID;
    bool any = false;
    for (int32_t c = 0; c < ncand; ++c) any |= eligible[c] != 0;
    if (!any) return PEPP_E_INVALID;
    *cand = pepp::history_pick(h, key, ncand, eligible, min_samples < 1 ? 1 : min_samples, calibrating, predicted_us);
    return PEPP_OK;
}

extern "C" PEPP_API pepp_status_t pepp_dist_choose(int32_t nranks, int32_t nd, const double* means,
                                                  const uint8_t* eligible, int32_t* choice, double* agreed) {
    if (nranks < 1 || nd < 1 || !means || !choice) return PEPP_E_INVALID;
    std::vector<double> ag(nd, 0.0);
    for (int32_t d = 0; d < nd; ++d) {
        double m = 0.0;
        for (int32_t r = 0; r < nranks; ++r) {
            const double v = means[(int64_t)r * nd + d];
            if (!(v >= 0.0)) return PEPP_E_INVALID;       // NaN or negative
            m = std::max(m, v);
        }
        ag[d] = m;
    }
    if (agreed) std::copy(ag.begin(), ag.end(), agreed);
    *choice = pepp::dist_argmin(nd, ag.data(), eligible);
    return *choice < 0 ? PEPP_E_STATE : PEPP_OK;
}

extern "C" PEPP_API pepp_status_t pepp_history_prior(const pepp_history* h, uint64_t key, int32_t n, const int32_t* ids,
                                                    double* prior, uint64_t* from_key) {
    if (!h || n < 0 || (n > 0 && (!ids || !prior))) return PEPP_E_INVALID;
    return pepp::history_prior(h, key, n, ids, prior, from_key) ? PEPP_OK : PEPP_E_STATE;
}

extern "C" PEPP_API pepp_status_t pepp_history_save(const pepp_history* h, const char* path) {
    if (!h || !path) return PEPP_E_INVALID;
    FILE* f = std::fopen(path, "w");
    if (!f) return PEPP_E_INVALID;
    std::fprintf(f, "# pepp_spmv history v1: key cand count mean_us m2\n");
    for (const auto& kv : h->table)
        std::fprintf(f, "%llu %d %lld %.17g %.17g\n", (unsigned long long)kv.first.key, kv.first.cand,
                     (long long)kv.second.count, kv.second.mean, kv.second.m2);
    std::fclose(f);
    return PEPP_OK;
}

extern "C" PEPP_API pepp_status_t pepp_history_load(pepp_history* h, const char* path) {
    if (!h || !path) return PEPP_E_INVALID;
    FILE* f = std::fopen(path, "r");
    if (!f) return PEPP_E_INVALID;
    char line[512];
    while (std::fgets(line, sizeof line, f)) {
        if (line[0] == '#') continue;
        unsigned long long key; int cand; long long cnt; double mean, m2;
        if (std::sscanf(line, "%llu %d %lld %lg %lg", &key, &cand, &cnt, &mean, &m2) == 5 && cnt > 0) {
            pepp::Welford& w = h->table[{(uint64_t)key, (int32_t)cand}];
            // merge (Chan et al. parallel Welford)
            const double n1 = (double)w.count, n2 = (double)cnt, n = n1 + n2;
            const double d = mean - w.mean;
            w.mean = (n1 * w.mean + n2 * mean) / n;
            w.m2 = w.m2 + m2 + d * d * n1 * n2 / n;
            w.count += cnt;
        }
    }
    std::fclose(f);
    return PEPP_OK;
}

extern "C" PEPP_API uint64_t pepp_context_key(int64_t nrows, int64_t ncols, int64_t nnz, double cv, int32_t nparts,
                                              int32_t instance) {
    return pepp::context_key(nrows, ncols, nnz, cv, nparts, instance);
}
