// planner.cpp -- host-side optimisers of mu-cuDNN (pure functions, no GPU).
//
//   mucu_plan_wr      WR dynamic program          (Sec. III-B)
//   mucu_pareto_front WD set-valued DP + pruning   (Sec. III-C1)
//   mucu_solve_wd     WD 0-1 ILP as exact MCKP     (Eq. (1)-(4))
//
// All arithmetic is integer (ns, bytes; reading G10), so results are exact and
// independent of evaluation order.  Tie-breaks follow readings G8/G11/G15/G17
// (DESIGN.md "Readings").  The brute-force reference these are tested against
// lives in oracle/planner_bf.py and shares nothing with this file.
#include <algorithm>
#include <cstdint>
#include <cstring>
#include <limits>
#include <new>
#include <vector>

#include "mucudnn.h"
#include "mucudnn_internal.h"

namespace mucu {

static const int64_t kInf = std::numeric_limits<int64_t>::max() / 4;

// Fastest micro-configuration for micro-batch b within `limit` (P:L88 step 1:
// "the fastest micro-configuration ... within the workspace constraint").
// Ties: smaller workspace, then smaller algorithm id (reading G11).
static bool best_micro(int32_t n, const int64_t* t, const uint64_t* ws, int32_t b, uint64_t limit,
                       int64_t* bt, uint64_t* bm, int32_t* ba) {
    bool found = false;
    for (int32_t a = 0; a < MUCU_NUM_ALGOS; ++a) {
        int64_t ti = t[(size_t)a * (n + 1) + b];
        uint64_t mi = ws[(size_t)a * (n + 1) + b];
        if (ti < 0 || mi > limit) continue;
        if (!found || ti < *bt || (ti == *bt && (mi < *bm || (mi == *bm && a < *ba)))) {
            *bt = ti; *bm = mi; *ba = a; found = true;
        }
    }
    return found;
}

}  // namespace mucu

using namespace mucu;

extern "C" mucu_status_t mucu_plan_wr(int32_t n, const int64_t* time_ns, const uint64_t* ws,
                                      uint64_t ws_limit, mucu_micro_config_t* out, int32_t cap,
                                      int32_t* count, int64_t* total_ns) {
    if (n <= 0 || !time_ns || !ws || !count) return set_error(MUCU_ERR_INVALID_VALUE, "plan_wr: bad arguments");
    // Step 1 result: T_mu(b), a_b.
    std::vector<int64_t> tmu(n + 1, -1);
    std::vector<int32_t> amu(n + 1, -1);
    for (int32_t b = 1; b <= n; ++b) {
        int64_t bt = 0; uint64_t bm = 0; int32_t ba = 0;
        if (best_micro(n, time_ns, ws, b, ws_limit, &bt, &bm, &ba)) { tmu[b] = bt; amu[b] = ba; }
    }
    // Step 2: T(b) = min(T_mu(b), min_{b'} T_mu(b') + T(b - b')), memoised.
    // Canonical tie-break (reading G8): minimise (T, #parts); among those take
    // the largest first part b', which yields parts in non-increasing order.
    std::vector<int64_t> T(n + 1, kInf);
    std::vector<int32_t> parts(n + 1, 0), first(n + 1, 0);
    T[0] = 0;
    for (int32_t b = 1; b <= n; ++b) {
        for (int32_t bp = b; bp >= 1; --bp) {  // descending: strict '<' keeps the largest b'
            if (tmu[bp] < 0 || T[b - bp] >= kInf) continue;
            int64_t cand = tmu[bp] + T[b - bp];
            int32_t cp = 1 + parts[b - bp];
            if (cand < T[b] || (cand == T[b] && cp < parts[b])) {
                T[b] = cand; parts[b] = cp; first[b] = bp;
            }
        }
    }
    if (T[n] >= kInf) return set_error(MUCU_ERR_INSUFFICIENT_WORKSPACE, "plan_wr: no configuration fits the workspace limit");
    // Step 3: output C(N).
    *count = parts[n];
    if (total_ns) *total_ns = T[n];
    if (!out || cap < parts[n]) return set_error(MUCU_ERR_CAPACITY, "plan_wr: output capacity too small");
    int32_t i = 0;
    for (int32_t b = n; b > 0; b -= first[b]) {
        out[i].algo = amu[first[b]];
        out[i].micro_n = first[b];
        ++i;
    }
    return MUCU_OK;
}

namespace {

// One configuration on a per-b front: cost and a back-pointer
// ([c] (+) C' with c = (algo, bp) and C' = front[b - bp][prev]).
struct FrontEntry {
    int64_t t;
    uint64_t m;
    int32_t bp, algo, prev, nparts;
};

}  // namespace

extern "C" mucu_status_t mucu_pareto_front(int32_t n, const int64_t* time_ns, const uint64_t* ws,
                                           uint64_t ws_cap, int64_t* front_t, uint64_t* front_m,
                                           int32_t cap, int32_t* front_len,
                                           mucu_micro_config_t* plans, int32_t* plan_len) {
    if (n <= 0 || !time_ns || !ws || !front_len) return set_error(MUCU_ERR_INVALID_VALUE, "pareto_front: bad arguments");
    try {
        std::vector<std::vector<FrontEntry>> F(n + 1);
        F[0].push_back({0, 0, 0, -1, -1, 0});
        std::vector<FrontEntry> cand;
        for (int32_t b = 1; b <= n; ++b) {
            cand.clear();
            // U_{b'} { [c] (+) C' : c in C_mu(b'), C' in C(b - b') }
            for (int32_t bp = 1; bp <= b; ++bp) {
                const std::vector<FrontEntry>& rest = F[b - bp];
                if (rest.empty()) continue;
                for (int32_t a = 0; a < MUCU_NUM_ALGOS; ++a) {
                    int64_t tc = time_ns[(size_t)a * (n + 1) + bp];
                    uint64_t mc = ws[(size_t)a * (n + 1) + bp];
                    if (tc < 0 || mc > ws_cap) continue;
                    for (int32_t j = 0; j < (int32_t)rest.size(); ++j) {
                        const FrontEntry& e = rest[j];
                        cand.push_back({tc + e.t, std::max(mc, e.m), bp, a, j, e.nparts + 1});
                    }
                }
            }
            // D(.): Pareto filter (reading G15) -- sort by M then T
            // and keep strictly decreasing T.  Among exact (T, M) ties the first
            // in a fixed deterministic order is kept.
            std::sort(cand.begin(), cand.end(), [](const FrontEntry& x, const FrontEntry& y) {
                if (x.m != y.m) return x.m < y.m;
                if (x.t != y.t) return x.t < y.t;
                if (x.nparts != y.nparts) return x.nparts < y.nparts;
                if (x.bp != y.bp) return x.bp > y.bp;
                if (x.algo != y.algo) return x.algo < y.algo;
                return x.prev < y.prev;
            });
            std::vector<FrontEntry>& out = F[b];
            for (const FrontEntry& e : cand)
                if (out.empty() || e.t < out.back().t) out.push_back(e);
        }
        const std::vector<FrontEntry>& fn = F[n];
        *front_len = (int32_t)fn.size();
        if (fn.empty()) return set_error(MUCU_ERR_INSUFFICIENT_WORKSPACE, "pareto_front: no configuration fits ws_cap");
        if (cap < (int32_t)fn.size()) return set_error(MUCU_ERR_CAPACITY, "pareto_front: capacity too small");
        for (int32_t i = 0; i < (int32_t)fn.size(); ++i) {
            if (front_t) front_t[i] = fn[i].t;
            if (front_m) front_m[i] = fn[i].m;
            if (plans && plan_len) {
                std::vector<mucu_micro_config_t> p;
                int32_t b = n, idx = i;
                while (b > 0) {
                    const FrontEntry& e = F[b][idx];
                    p.push_back({e.algo, e.bp});
                    idx = e.prev;
                    b -= e.bp;
                }
                std::stable_sort(p.begin(), p.end(), [](const mucu_micro_config_t& x, const mucu_micro_config_t& y) {
                    return x.micro_n > y.micro_n;
                });
                plan_len[i] = (int32_t)p.size();
                std::memcpy(plans + (size_t)i * n, p.data(), p.size() * sizeof(mucu_micro_config_t));
            }
        }
        return MUCU_OK;
    } catch (const std::bad_alloc&) {
        return set_error(MUCU_ERR_INTERNAL, "pareto_front: out of host memory");
    }
}

namespace {

struct KState {
    int64_t t;
    uint64_t m;
    int32_t prev;    // index into previous level's kept states
    int32_t choice;  // option index of this kernel
    int32_t lex;     // rank of the prefix choice vector among this level's states
};

}  // namespace

static inline uint64_t align256(uint64_t m) { return (m + 255u) & ~uint64_t(255u); }

extern "C" mucu_status_t mucu_solve_wd(int32_t num_kernels, const int32_t* front_len, const int64_t* t,
                                       const uint64_t* m, uint64_t total_limit, int32_t* choice,
                                       uint64_t* offset, int64_t* total_ns) {
    if (num_kernels <= 0 || !front_len || !t || !m || !choice)
        return set_error(MUCU_ERR_INVALID_VALUE, "solve_wd: bad arguments");
    try {
        std::vector<size_t> off(num_kernels + 1, 0);
        for (int32_t k = 0; k < num_kernels; ++k) {
            if (front_len[k] <= 0) return set_error(MUCU_ERR_INVALID_VALUE, "solve_wd: empty option list");
            off[k + 1] = off[k] + (size_t)front_len[k];
        }
        // Minimal remaining workspace after kernel k (budget pruning).
        std::vector<uint64_t> minrest(num_kernels + 1, 0);
        for (int32_t k = num_kernels - 1; k >= 0; --k) {
            uint64_t mn = std::numeric_limits<uint64_t>::max();
            for (size_t i = off[k]; i < off[k + 1]; ++i) mn = std::min(mn, align256(m[i]));
            minrest[k] = minrest[k + 1] + mn;
        }
        if (minrest[0] > total_limit)
            return set_error(MUCU_ERR_INFEASIBLE, "solve_wd: total limit below the sum of minimal workspaces");
        // Exact MCKP by Pareto merging (Nemhauser-Ullmann): after kernel k keep
        // every non-dominated (sum M, sum T) prefix; a dominated prefix can never
        // complete to an optimum (same argument as the pruning proof).
        std::vector<std::vector<KState>> L(num_kernels + 1);
        L[0].push_back({0, 0, -1, -1, 0});
        std::vector<KState> cand;
        for (int32_t k = 0; k < num_kernels; ++k) {
            const std::vector<KState>& S = L[k];
            cand.clear();
            for (int32_t s = 0; s < (int32_t)S.size(); ++s) {
                for (size_t i = off[k]; i < off[k + 1]; ++i) {
                    uint64_t mm = S[s].m + align256(m[i]);
                    if (mm + minrest[k + 1] > total_limit) continue;
                    cand.push_back({S[s].t + t[i], mm, s, (int32_t)(i - off[k]), 0});
                }
            }
            // Lexicographic order of a prefix = (lex rank of its parent, choice).
            std::sort(cand.begin(), cand.end(), [&S](const KState& x, const KState& y) {
                if (x.m != y.m) return x.m < y.m;
                if (x.t != y.t) return x.t < y.t;
                int32_t lx = S[x.prev].lex, ly = S[y.prev].lex;
                if (lx != ly) return lx < ly;
                return x.choice < y.choice;
            });
            std::vector<KState>& out = L[k + 1];
            for (const KState& c : cand)
                if (out.empty() || c.t < out.back().t) out.push_back(c);
            // Rank the kept prefixes lexicographically for the next level.
            std::vector<int32_t> order(out.size());
            for (size_t i = 0; i < order.size(); ++i) order[i] = (int32_t)i;
            std::sort(order.begin(), order.end(), [&](int32_t a, int32_t b) {
                int32_t la = S[out[a].prev].lex, lb = S[out[b].prev].lex;
                if (la != lb) return la < lb;
                return out[a].choice < out[b].choice;
            });
            for (size_t r = 0; r < order.size(); ++r) out[order[r]].lex = (int32_t)r;
            if (out.empty()) return set_error(MUCU_ERR_INFEASIBLE, "solve_wd: infeasible");
        }
        // Optimum: minimal sum T (the last Pareto point, T strictly decreasing in M).
        const std::vector<KState>& last = L[num_kernels];
        int32_t idx = (int32_t)last.size() - 1;
        if (total_ns) *total_ns = last[idx].t;
        for (int32_t k = num_kernels; k >= 1; --k) {
            const KState& st = L[k][idx];
            choice[k - 1] = st.choice;
            idx = st.prev;
        }
        if (offset) {
            uint64_t o = 0;
            for (int32_t k = 0; k < num_kernels; ++k) {
                offset[k] = o;
                o += align256(m[off[k] + choice[k]]);
            }
        }
        return MUCU_OK;
    } catch (const std::bad_alloc&) {
        return set_error(MUCU_ERR_INTERNAL, "solve_wd: out of host memory");
    }
}
