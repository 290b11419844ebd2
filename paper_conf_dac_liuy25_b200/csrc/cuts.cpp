// cuts.cpp — host cut generator for local function checking (§III-C1, :132-154).
//
// Priority cuts by cut enumeration, Eq. (1):
//   E(n) = { u | v : u in P(n0) + {{n0}}, v in P(n1) + {{n1}}, |u | v| <= k_l },
// P(n) = the C best cuts of E(n) after dropping dominated cuts (supersets of another candidate,
// priority cuts of ref. [27]), ranked by the Table I order of the pass:
//   pass 0: large average fanout > small size > small average level
//   pass 1: small average level > small size > large average fanout
//   pass 2: large average level > small size > large average fanout
// Non-representatives rank first by similarity to their representative's priority cuts,
// s(c, P) = sum_{c' in P} |c & c'| / |c | c'|. Nodes are visited in increasing id,
// a topological order in which every representative (minimum id of its class) precedes its
// members — the property the enumeration levels of Eq. (2) provide in the paper's level-wise GPU
// schedule. Common cuts of a pair (repr r, member m) are {u | v : u in P(r), v in P(m),
// |u | v| <= k_l} without trivial cuts (reading Q14), smallest first.
//
// This is the host-minimal stand-in for the paper's GPU cut generator;
// the checks themselves run on the GPU through cec_check_local_cuts.
#include <algorithm>
#include <chrono>
#include <cstdio>
#include <atomic>
#include <functional>
#include <memory>
#include <mutex>
#include <condition_variable>
#include <thread>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "cec_ctx.hpp"

namespace {

constexpr int KMAX = 24;

struct Cut {
    uint8_t n = 0;
    uint32_t leaf[KMAX];
    uint64_t sig = 0;  // bloom signature for fast subset tests
    // ranking metrics (integers: exact comparisons)
    uint64_t sum_fanout = 0, sum_level = 0;
    unsigned __int128 sim = 0;  // similarity x lcm(1..2*KMAX): exact, so ties are unambiguous
};

unsigned __int128 lcm_upto(int n) {
    unsigned __int128 l = 1;
    for (int i = 2; i <= n; ++i) {
        unsigned __int128 a = l, b = (unsigned __int128)i;
        while (b) {
            unsigned __int128 t = a % b;
            a = b;
            b = t;
        }
        l = l / a * (unsigned __int128)i;
    }
    return l;
}

inline uint64_t bit_of(uint32_t id) { return 1ull << (id & 63); }

// merge sorted leaf lists; false if the union exceeds k
bool merge(const uint32_t *a, int na, const uint32_t *b, int nb, int k, Cut &out) {
    int i = 0, j = 0, n = 0;
    while (i < na || j < nb) {
        uint32_t v;
        if (j >= nb || (i < na && a[i] < b[j])) {
            v = a[i++];
        } else if (i >= na || b[j] < a[i]) {
            v = b[j++];
        } else {
            v = a[i++];
            ++j;
        }
        if (n == k) return false;
        out.leaf[n++] = v;
    }
    out.n = (uint8_t)n;
    out.sig = 0;
    for (int t = 0; t < n; ++t) out.sig |= bit_of(out.leaf[t]);
    return true;
}

bool subset(const Cut &small, const Cut &big) {  // small ⊆ big
    if ((small.sig & ~big.sig) != 0 || small.n > big.n) return false;
    int j = 0;
    for (int i = 0; i < small.n; ++i) {
        while (j < big.n && big.leaf[j] < small.leaf[i]) ++j;
        if (j == big.n || big.leaf[j] != small.leaf[i]) return false;
        ++j;
    }
    return true;
}

int inter(const Cut &a, const Cut &b) {
    int i = 0, j = 0, c = 0;
    while (i < a.n && j < b.n) {
        if (a.leaf[i] == b.leaf[j]) {
            ++c;
            ++i;
            ++j;
        } else if (a.leaf[i] < b.leaf[j]) {
            ++i;
        } else {
            ++j;
        }
    }
    return c;
}

bool same(const Cut &a, const Cut &b) {
    return a.n == b.n && a.sig == b.sig && std::memcmp(a.leaf, b.leaf, a.n * sizeof(uint32_t)) == 0;
}

// a < b in the Table I order of the pass (cross-multiplied averages: exact)
bool table1_less(const Cut &a, const Cut &b, int pass) {
    const uint64_t fa = a.sum_fanout * b.n, fb = b.sum_fanout * a.n;  // avg fanout a vs b
    const uint64_t la = a.sum_level * b.n, lb = b.sum_level * a.n;    // avg level a vs b
    if (pass == 0) {
        if (fa != fb) return fa > fb;
        if (a.n != b.n) return a.n < b.n;
        if (la != lb) return la < lb;
    } else if (pass == 1) {
        if (la != lb) return la < lb;
        if (a.n != b.n) return a.n < b.n;
        if (fa != fb) return fa > fb;
    } else {
        if (la != lb) return la > lb;
        if (a.n != b.n) return a.n < b.n;
        if (fa != fb) return fa > fb;
    }
    return std::lexicographical_compare(a.leaf, a.leaf + a.n, b.leaf, b.leaf + b.n);
}

Cut trivial_cut(uint32_t id) {  // the constant needs no leaf: its cut is empty
    Cut t;
    if (id == 0) return t;
    t.n = 1;
    t.leaf[0] = id;
    t.sig = bit_of(id);
    return t;
}

struct CutJob {  // shared, read-only inputs of the per-node enumeration
    const cec_ctx *c;
    const std::vector<uint32_t> *fanout, *repr_of;
    uint32_t k_l, C;
    int pass;
};

// Fast path of node_cuts: the leaves of every candidate cut of n are drawn from the leaves of
// P(n0) + {{n0}} and P(n1) + {{n1}}; when that dictionary has <= 128 node ids, a cut is a 128-bit
// mask over it (dictionary sorted by id) and every operation of Eq. (1) and the ranking is exact
// bit arithmetic: union = OR, |cut| = popcount, subset = (x & ~y) == 0, and for two cuts of EQUAL
// size the lexicographic order of their sorted leaf lists is decided by the lowest node of their
// symmetric difference (the list holding it is the smaller one: every smaller node is in both).
// Same candidates, same order relations, same result as the list path below (pinned by
// tests/test_driver_host.py against oracle/cuts.py); returns false when the dictionary is larger.
typedef unsigned __int128 u128;
inline int pop128(u128 x) { return __builtin_popcountll((uint64_t)x) + __builtin_popcountll((uint64_t)(x >> 64)); }
inline int ctz128(u128 x) {
    const uint64_t lo = (uint64_t)x;
    return lo ? __builtin_ctzll(lo) : 64 + __builtin_ctzll((uint64_t)(x >> 64));
}
inline bool lex_less_masks(u128 x, u128 y) {  // equal popcounts; sorted leaf lists x < y
    const u128 d = x ^ y;
    return d != 0 && ((x >> ctz128(d)) & 1) != 0;
}

bool node_cuts_masks(const CutJob &J, uint32_t id, std::vector<std::vector<Cut>> &P) {
    const cec_ctx *c = J.c;
    const uint32_t a = c->f0[id] >> 1, b = c->f1[id] >> 1;
    const std::vector<Cut> &Pa = P[a], &Pb = P[b];
    const Cut ta = trivial_cut(a), tb = trivial_cut(b);
    // thread_local scratch bound to plain references once: every access of a thread_local in a
    // shared library is a __tls_get_addr call, which dominated the sort comparators
    thread_local std::vector<uint32_t> tD;
    thread_local std::vector<u128> tma, tmb, tE;
    thread_local std::vector<uint8_t> tEn;
    thread_local std::vector<uint32_t> tord, tkept, trk;
    thread_local std::vector<uint64_t> tdfan, tdlev;
    thread_local std::vector<Cut> tK;
    std::vector<uint32_t> &D = tD, &ord = tord, &kept = tkept, &rk = trk;
    std::vector<u128> &ma = tma, &mb = tmb, &E = tE;
    std::vector<uint8_t> &En = tEn;
    std::vector<uint64_t> &dfan = tdfan, &dlev = tdlev;
    std::vector<Cut> &K = tK;
    D.clear();
    for (const std::vector<Cut> *L : {&Pa, &Pb})
        for (const Cut &u : *L) D.insert(D.end(), u.leaf, u.leaf + u.n);
    D.insert(D.end(), ta.leaf, ta.leaf + ta.n);
    D.insert(D.end(), tb.leaf, tb.leaf + tb.n);
    std::sort(D.begin(), D.end());
    D.erase(std::unique(D.begin(), D.end()), D.end());
    if (D.size() > 128) return false;
    auto mask_of = [&](const Cut &u) {
        u128 m = 0;
        for (int t = 0; t < u.n; ++t) m |= (u128)1 << (std::lower_bound(D.begin(), D.end(), u.leaf[t]) - D.begin());
        return m;
    };
    ma.clear();
    mb.clear();
    for (const Cut &u : Pa) ma.push_back(mask_of(u));
    ma.push_back(mask_of(ta));
    for (const Cut &v : Pb) mb.push_back(mask_of(v));
    mb.push_back(mask_of(tb));
    // Eq. (1) candidates in the list path's order; drop the empty cut and the trivial cut {n}
    // (n itself is never in the dictionary: every leaf id is below id)
    E.clear();
    En.clear();
    for (u128 u : ma)
        for (u128 v : mb) {
            const u128 m = u | v;
            const int n = pop128(m);
            if (n > (int)J.k_l || n == 0) continue;
            E.push_back(m);
            En.push_back((uint8_t)n);
        }
    // Dominance filter: the kept set is the set of minimal candidates (no kept cut is a subset of
    // another), which does not depend on the order inside one size class, only on visiting smaller
    // sizes first; the final Table I / similarity ranking below is a total order. So candidates are
    // bucketed by size (counting sort) and, inside a bucket, sorted by mask value only to find
    // repeats; a candidate is checked against kept cuts of strictly smaller size (two different
    // cuts of one size are never subsets of each other).
    uint32_t bstart[KMAX + 2] = {0};
    for (uint8_t n : En) ++bstart[n + 1];
    for (int b = 0; b <= KMAX; ++b) bstart[b + 1] += bstart[b];
    ord.resize(E.size());
    {
        uint32_t fillp[KMAX + 1];
        for (int b = 0; b <= KMAX; ++b) fillp[b] = bstart[b];
        for (uint32_t i = 0; i < E.size(); ++i) ord[fillp[En[i]]++] = i;
    }
    kept.clear();
    for (int b = 1; b <= (int)J.k_l && b <= KMAX; ++b) {
        const uint32_t lo = bstart[b], hi = bstart[b + 1];
        if (lo == hi) continue;
        std::sort(ord.begin() + lo, ord.begin() + hi, [&](uint32_t xi, uint32_t yi) { return E[xi] < E[yi]; });
        const size_t smaller = kept.size();  // kept cuts of size < b
        for (uint32_t t = lo; t < hi; ++t) {
            const u128 x = E[ord[t]];
            if (t > lo && x == E[ord[t - 1]]) continue;  // a repeat of the previous candidate
            bool dom = false;
            for (size_t q = 0; q < smaller; ++q)
                if ((E[kept[q]] & ~x) == 0) {
                    dom = true;
                    break;
                }
            if (!dom) kept.push_back(ord[t]);
        }
    }
    // metrics per dictionary entry
    dfan.resize(D.size());
    dlev.resize(D.size());
    for (size_t i = 0; i < D.size(); ++i) {
        dfan[i] = (*J.fanout)[D[i]];
        dlev[i] = c->level[D[i]];
    }
    K.resize(kept.size());
    for (size_t t = 0; t < kept.size(); ++t) {
        Cut &x = K[t];
        u128 m = E[kept[t]];
        x.n = 0;
        x.sig = 0;
        x.sum_fanout = x.sum_level = 0;
        x.sim = 0;
        while (m) {
            const int i = ctz128(m);
            m &= m - 1;
            x.leaf[x.n++] = D[i];
            x.sig |= bit_of(D[i]);
            x.sum_fanout += dfan[i];
            x.sum_level += dlev[i];
        }
    }
    rk.resize(K.size());
    for (uint32_t i = 0; i < rk.size(); ++i) rk[i] = i;
    const uint32_t r = (*J.repr_of)[id];
    if (r != 0xFFFFFFFFu && !P[r].empty()) {
        static const unsigned __int128 L = lcm_upto(2 * KMAX);
        for (Cut &x : K) {
            unsigned __int128 sv = 0;
            for (const Cut &y : P[r]) {
                const int in = inter(x, y);
                sv += (unsigned __int128)in * (L / (unsigned __int128)(x.n + y.n - in));
            }
            x.sim = sv;
        }
        std::sort(rk.begin(), rk.end(), [&](uint32_t xi, uint32_t yi) {
            const Cut &x = K[xi], &y = K[yi];
            if (x.sim != y.sim) return x.sim > y.sim;
            return table1_less(x, y, J.pass);
        });
    } else {
        std::sort(rk.begin(), rk.end(), [&](uint32_t xi, uint32_t yi) { return table1_less(K[xi], K[yi], J.pass); });
    }
    std::vector<Cut> out;
    out.reserve(std::min<size_t>(rk.size(), J.C));
    for (size_t t = 0; t < rk.size() && t < J.C; ++t) out.push_back(K[rk[t]]);
    P[id].swap(out);
    return true;
}

// P(id) from P(fanins) (and P(repr) for a member): Eq. (1), dominance, Table I / similarity order.
void node_cuts(const CutJob &J, uint32_t id, std::vector<std::vector<Cut>> &P) {
    static const bool lists_only = getenv("CEC_CUTS_LISTS") != nullptr;  // the list path (A/B, tests)
    if (!lists_only && node_cuts_masks(J, id, P)) return;
    const cec_ctx *c = J.c;
    const uint32_t a = c->f0[id] >> 1, b = c->f1[id] >> 1;
    const std::vector<Cut> &Pa = P[a], &Pb = P[b];
    const Cut ta = trivial_cut(a), tb = trivial_cut(b);
    // candidates in the order P(n0) + {{n0}} x P(n1) + {{n1}}; ranked through index arrays (a Cut
    // is ~150 bytes: sorting the objects themselves dominated the enumeration)
    thread_local std::vector<Cut> tE;
    thread_local std::vector<uint32_t> tord, tkept;
    std::vector<Cut> &E = tE;
    std::vector<uint32_t> &ord = tord, &kept = tkept;
    E.clear();
    Cut m;
    for (size_t i = 0; i <= Pa.size(); ++i) {
        const Cut &u = i < Pa.size() ? Pa[i] : ta;
        for (size_t j = 0; j <= Pb.size(); ++j) {
            const Cut &v = j < Pb.size() ? Pb[j] : tb;
            // more distinct signature bits than k_l means more than k_l distinct leaves
            if (__builtin_popcountll(u.sig | v.sig) > (int)J.k_l) continue;
            if (merge(u.leaf, u.n, v.leaf, v.n, (int)J.k_l, m)) {
                if (m.n == 0 || (m.n == 1 && m.leaf[0] == id)) continue;
                E.push_back(m);
            }
        }
    }
    // dedupe + drop dominated: process by size, keep a cut unless a kept cut is its subset
    ord.resize(E.size());
    for (uint32_t i = 0; i < ord.size(); ++i) ord[i] = i;
    std::sort(ord.begin(), ord.end(), [&](uint32_t xi, uint32_t yi) {
        const Cut &x = E[xi], &y = E[yi];
        if (x.n != y.n) return x.n < y.n;
        return std::lexicographical_compare(x.leaf, x.leaf + x.n, y.leaf, y.leaf + y.n);
    });
    kept.clear();
    for (uint32_t xi : ord) {
        const Cut &x = E[xi];
        bool dom = false;
        for (uint32_t ki : kept) {
            const Cut &k = E[ki];
            if (same(k, x) || subset(k, x)) {
                dom = true;
                break;
            }
        }
        if (!dom) kept.push_back(xi);
    }
    for (uint32_t xi : kept) {
        Cut &x = E[xi];
        x.sum_fanout = x.sum_level = 0;
        for (int t = 0; t < x.n; ++t) {
            x.sum_fanout += (*J.fanout)[x.leaf[t]];
            x.sum_level += c->level[x.leaf[t]];
        }
        x.sim = 0;
    }
    const uint32_t r = (*J.repr_of)[id];
    if (r != 0xFFFFFFFFu && !P[r].empty()) {
        static const unsigned __int128 L = lcm_upto(2 * KMAX);
        for (uint32_t xi : kept) {
            Cut &x = E[xi];
            unsigned __int128 sv = 0;
            for (const Cut &y : P[r]) {
                const int in = inter(x, y);
                sv += (unsigned __int128)in * (L / (unsigned __int128)(x.n + y.n - in));
            }
            x.sim = sv;
        }
        std::sort(kept.begin(), kept.end(), [&](uint32_t xi, uint32_t yi) {
            const Cut &x = E[xi], &y = E[yi];
            if (x.sim != y.sim) return x.sim > y.sim;
            return table1_less(x, y, J.pass);
        });
    } else {
        std::sort(kept.begin(), kept.end(), [&](uint32_t xi, uint32_t yi) { return table1_less(E[xi], E[yi], J.pass); });
    }
    std::vector<Cut> out;
    out.reserve(std::min<size_t>(kept.size(), J.C));
    for (size_t t = 0; t < kept.size() && t < J.C; ++t) out.push_back(E[kept[t]]);
    P[id].swap(out);
}

// common cuts u|v of a pair (no trivial cuts, <= k_l leaves), smallest first, at most max_cuts
// Mask path of common_cuts_of (the same dictionary trick as node_cuts_masks): unions by OR, size by
// popcount, (size, lexicographic) order by lex_less_masks, repeats adjacent after the sort; only the
// first max_cuts survivors are turned back into leaf lists. False when > 128 distinct leaves.
bool common_cuts_masks(const std::vector<std::vector<Cut>> &P, uint32_t r, uint32_t mbr, uint32_t k_l,
                       uint32_t max_cuts, std::vector<Cut> &common) {
    thread_local std::vector<uint32_t> tD;
    thread_local std::vector<u128> tmr, tmm, tE;
    thread_local std::vector<uint8_t> tEn;
    thread_local std::vector<uint32_t> tord;
    std::vector<uint32_t> &D = tD, &ord = tord;
    std::vector<u128> &mr = tmr, &mm = tmm, &E = tE;
    std::vector<uint8_t> &En = tEn;
    D.clear();
    for (const std::vector<Cut> *L : {&P[r], &P[mbr]})
        for (const Cut &u : *L) D.insert(D.end(), u.leaf, u.leaf + u.n);
    std::sort(D.begin(), D.end());
    D.erase(std::unique(D.begin(), D.end()), D.end());
    if (D.size() > 128) return false;
    auto mask_of = [&](const Cut &u) {
        u128 m = 0;
        for (int t = 0; t < u.n; ++t) m |= (u128)1 << (std::lower_bound(D.begin(), D.end(), u.leaf[t]) - D.begin());
        return m;
    };
    mr.clear();
    mm.clear();
    for (const Cut &u : P[r]) mr.push_back(mask_of(u));
    for (const Cut &v : P[mbr]) mm.push_back(mask_of(v));
    E.clear();
    En.clear();
    for (u128 u : mr)
        for (u128 v : mm) {
            const u128 m = u | v;
            const int n = pop128(m);
            if (n == 0 || n > (int)k_l) continue;
            E.push_back(m);
            En.push_back((uint8_t)n);
        }
    ord.resize(E.size());
    for (uint32_t i = 0; i < ord.size(); ++i) ord[i] = i;
    std::sort(ord.begin(), ord.end(), [&](uint32_t xi, uint32_t yi) {
        if (En[xi] != En[yi]) return En[xi] < En[yi];
        return lex_less_masks(E[xi], E[yi]);
    });
    common.clear();
    for (size_t t = 0; t < ord.size() && common.size() < max_cuts; ++t) {
        if (t > 0 && E[ord[t]] == E[ord[t - 1]]) continue;
        Cut x;
        u128 m = E[ord[t]];
        while (m) {
            const int i = ctz128(m);
            m &= m - 1;
            x.leaf[x.n++] = D[i];
            x.sig |= bit_of(D[i]);
        }
        common.push_back(x);
    }
    return true;
}

void common_cuts_of(const std::vector<std::vector<Cut>> &P, uint32_t r, uint32_t mbr, uint32_t k_l, uint32_t max_cuts,
                    std::vector<Cut> &common) {
    static const bool lists_only = getenv("CEC_CUTS_LISTS") != nullptr;
    if (!lists_only && common_cuts_masks(P, r, mbr, k_l, max_cuts, common)) return;
    common.clear();
    Cut m;
    for (const Cut &u : P[r])
        for (const Cut &v : P[mbr])
            if (__builtin_popcountll(u.sig | v.sig) <= (int)k_l && merge(u.leaf, u.n, v.leaf, v.n, (int)k_l, m) &&
                m.n > 0)
                common.push_back(m);
    std::sort(common.begin(), common.end(), [](const Cut &x, const Cut &y) {
        if (x.n != y.n) return x.n < y.n;
        return std::lexicographical_compare(x.leaf, x.leaf + x.n, y.leaf, y.leaf + y.n);
    });
    common.erase(std::unique(common.begin(), common.end(), same), common.end());
    if (common.size() > max_cuts) common.resize(max_cuts);
}

// fanouts over the whole AIG (Table I metric), the TFI of the pair nodes (need), repr_of[member]
void cut_inputs(const cec_ctx *c, uint32_t npairs, const uint32_t *repr, const uint32_t *member,
                std::vector<uint32_t> &fanout, std::vector<uint8_t> &need, std::vector<uint32_t> &repr_of) {
    const uint32_t N = c->N();
    fanout.assign(N, 0);
    for (uint32_t id = c->I + 1; id < N; ++id) {
        ++fanout[c->f0[id] >> 1];
        ++fanout[c->f1[id] >> 1];
    }
    need.assign(N, 0);
    std::vector<uint32_t> st;
    for (uint32_t q = 0; q < npairs; ++q)
        for (uint32_t r : {repr[q], member[q]})
            if (!need[r]) {
                need[r] = 1;
                st.push_back(r);
            }
    while (!st.empty()) {
        const uint32_t v = st.back();
        st.pop_back();
        if (v <= c->I) continue;
        for (uint32_t f : {c->f0[v] >> 1, c->f1[v] >> 1})
            if (!need[f]) {
                need[f] = 1;
                st.push_back(f);
            }
    }
    repr_of.assign(N, 0xFFFFFFFFu);
    for (uint32_t q = 0; q < npairs; ++q) repr_of[member[q]] = repr[q];
}

}  // namespace

extern "C" cec_status cec_common_cuts(cec_ctx *c, uint32_t npairs, const uint32_t *repr, const uint32_t *member,
                                      uint32_t k_l, uint32_t C, int32_t pass_id, uint32_t max_cuts,
                                      uint32_t *pair_cut_off, uint32_t *cut_off, uint32_t *leaves) {
    if (!c || (npairs && (!repr || !member || !pair_cut_off || !cut_off || !leaves)) || k_l == 0 || k_l > KMAX ||
        C == 0 || max_cuts == 0 || pass_id < 0 || pass_id > 2)
        return CEC_E_ARG;
    const uint32_t N = c->N();
    for (uint32_t q = 0; q < npairs; ++q)
        if (repr[q] >= N || member[q] >= N || repr[q] >= member[q]) return CEC_E_ARG;
    std::vector<uint32_t> fanout, repr_of;
    std::vector<uint8_t> need;
    cut_inputs(c, npairs, repr, member, fanout, need, repr_of);
    size_t n_need = 0;
    for (uint32_t id = c->I + 1; id < N; ++id) n_need += need[id];
    // GPU generator for large cones (one launch per enumeration level pays off only at scale);
    // CEC_CUTS_GPU=1 / CEC_CUTS_HOST=1 force a side (tests pin both against oracle/cuts.py)
    const bool force_gpu = getenv("CEC_CUTS_GPU") != nullptr, force_host = getenv("CEC_CUTS_HOST") != nullptr;
    if (!c->host_only && C <= gpu_cuts_max_C() && !force_host && (force_gpu || n_need >= 20000)) {
        // GPU cut generator: nodes grouped by enumeration level (Eq. 2)
        cec_status st = cec_ensure_device_aig(c);
        if (st != CEC_OK) return st;
        std::vector<uint32_t> el(N, 0), pis;
        std::vector<std::vector<uint32_t>> lists;
        for (uint32_t id = 1; id <= c->I; ++id)
            if (need[id]) pis.push_back(id);
        for (uint32_t id = c->I + 1; id < N; ++id) {
            if (!need[id]) continue;
            uint32_t e = 1 + std::max(el[c->f0[id] >> 1], el[c->f1[id] >> 1]);
            if (repr_of[id] != 0xFFFFFFFFu) e = std::max(e, 1 + el[repr_of[id]]);
            el[id] = e;
            if (lists.size() <= e) lists.resize(e + 1);
            lists[e].push_back(id);
        }
        std::vector<uint32_t> lvl(c->level.begin(), c->level.end());
        std::vector<uint32_t> R(repr, repr + npairs), M(member, member + npairs), counts, flat;
        const char *e = gpu_common_cuts(c->d_f0, c->d_f1, N, fanout, lvl, repr_of, pis, lists, R, M, k_l, C, pass_id,
                                        max_cuts, c->stream, c->num_sms, counts, flat);
        if (e) {
            c->err = std::string("CUDA: ") + e + " (GPU cut generator)";
            return CEC_E_CUDA;
        }
        uint32_t ncut = 0, nleaf = 0;
        size_t pos = 0;
        cut_off[0] = 0;
        for (uint32_t q = 0; q < npairs; ++q) {
            pair_cut_off[q] = ncut;
            for (uint32_t t = 0; t < counts[q]; ++t) {
                const uint32_t n = flat[pos++];
                for (uint32_t i = 0; i < n; ++i) leaves[nleaf++] = flat[pos++];
                cut_off[++ncut] = nleaf;
            }
        }
        pair_cut_off[npairs] = ncut;
        return CEC_OK;
    }
    std::vector<std::vector<Cut>> P(N);
    for (uint32_t id = 1; id <= c->I; ++id)
        if (need[id]) P[id].push_back(trivial_cut(id));
    if (need[0]) P[0].push_back(trivial_cut(0));
    const CutJob J{c, &fanout, &repr_of, k_l, C, pass_id};
    for (uint32_t id = c->I + 1; id < N; ++id)
        if (need[id]) node_cuts(J, id, P);
    // common cuts per pair
    uint32_t ncut = 0, nleaf = 0;
    cut_off[0] = 0;
    std::vector<Cut> common;
    for (uint32_t q = 0; q < npairs; ++q) {
        pair_cut_off[q] = ncut;
        common_cuts_of(P, repr[q], member[q], k_l, max_cuts, common);
        for (const Cut &x : common) {
            for (int t = 0; t < x.n; ++t) leaves[nleaf++] = x.leaf[t];
            cut_off[++ncut] = nleaf;
        }
    }
    pair_cut_off[npairs] = ncut;
    return CEC_OK;
}

// ------------------------------------------------------------------------------------------------
// Alg. 2: one cut generation + checking pass with a common-cut buffer.
// Nodes are processed by enumeration level el (Eq. 2: el(PI) = 0, el(n) = 1 + max over the
// fanins, and above el(repr) for a non-representative), the nodes of one level in parallel on the
// host threads (they depend only on lower levels). When a member's priority cuts are ready, the
// common cuts of its pair go into the buffer (Alg. 2 l.11-12); a full buffer is flushed to the
// local-check kernels (Alg. 2 l.13-18, l.15 "Alg. 1 in local mode"), asynchronously: the GPU checks
// one buffer while the host enumerates the next levels. Per-pair results equal cec_common_cuts
// followed by cec_check_local_cuts on the same cuts (the cuts do not depend on the buffering).
// ------------------------------------------------------------------------------------------------
extern "C" cec_status cec_local_pass(cec_ctx *c, uint32_t npairs, const uint32_t *repr, const uint32_t *member,
                                     const uint8_t *phase, uint32_t k_l, uint32_t C, int32_t pass_id,
                                     uint32_t max_cuts, uint32_t buffer_checks, int32_t *verdict_out,
                                     uint32_t *num_checks_out, uint32_t *check_pair, uint32_t *check_cut_off,
                                     uint32_t *check_leaves, int32_t *check_verdict) {
    if (!c || (npairs && (!repr || !member || !phase || !verdict_out)) || !num_checks_out || k_l == 0 || k_l > KMAX ||
        C == 0 || max_cuts == 0 || pass_id < 0 || pass_id > 2)
        return CEC_E_ARG;
    const uint32_t N = c->N();
    for (uint32_t q = 0; q < npairs; ++q)
        if (repr[q] >= N || member[q] >= N || repr[q] >= member[q] || member[q] <= c->I) {
            c->err = "pair " + std::to_string(q) + ": need repr < member and member an AND node";
            return CEC_E_ARG;
        }
    if (c->host_only) {
        c->err = "host-only context: no CUDA device (no CPU fallback)";
        return CEC_E_CUDA;
    }
    std::vector<uint32_t> fanout, repr_of;
    std::vector<uint8_t> need;
    cut_inputs(c, npairs, repr, member, fanout, need, repr_of);
    // enumeration levels (Eq. 2) of the needed AND nodes
    std::vector<uint32_t> el(N, 0);
    std::vector<std::vector<uint32_t>> lists;
    for (uint32_t id = c->I + 1; id < N; ++id) {
        if (!need[id]) continue;
        uint32_t e = 1 + std::max(el[c->f0[id] >> 1], el[c->f1[id] >> 1]);
        if (repr_of[id] != 0xFFFFFFFFu) e = std::max(e, 1 + el[repr_of[id]]);
        el[id] = e;
        if (lists.size() <= e) lists.resize(e + 1);
        lists[e].push_back(id);
    }
    std::vector<std::vector<uint32_t>> pairs_at(lists.size());
    for (uint32_t q = 0; q < npairs; ++q) pairs_at[el[member[q]]].push_back(q);
    std::vector<std::vector<Cut>> P(N);
    for (uint32_t id = 1; id <= c->I; ++id)
        if (need[id]) P[id].push_back(trivial_cut(id));
    if (need[0]) P[0].push_back(trivial_cut(0));
    const CutJob J{c, &fanout, &repr_of, k_l, C, pass_id};
    WorkPool &pool = c->workers();
    for (uint32_t q = 0; q < npairs; ++q) verdict_out[q] = CEC_UNDECIDED;
    // the buffer: checks (pair, leaves) waiting for a flush; in-flight: one launched flush
    struct Flush {
        std::vector<uint32_t> pair, off{0}, leaves, la, lb;
        std::unique_ptr<cec_plan> plan;
        std::vector<int32_t> v;
    };
    Flush buf, inflight;
    uint32_t nchecks = 0;
    std::vector<uint32_t> log_pair, log_off{0}, log_leaves;  // every issued check, in issue order
    auto collect = [&](Flush &F) -> cec_status {
        if (!F.plan) return CEC_OK;
        F.v.assign(F.pair.size(), CEC_UNDECIDED);
        cec_status st = local_checks_collect(c, F.plan.get(), F.v.data());
        F.plan.reset();
        if (st != CEC_OK) return st;
        for (size_t t = 0; t < F.pair.size(); ++t)
            if (F.v[t] == CEC_EQUIVALENT) verdict_out[F.pair[t]] = CEC_EQUIVALENT;  // any cut proves the pair
        return CEC_OK;
    };
    std::vector<int32_t> all_v;  // verdicts of every issued check, in issue order
    auto launch = [&](Flush &F) -> cec_status {
        if (F.pair.empty()) return CEC_OK;
        uint32_t bad = 0, first_bad = 0;
        cec_status st = local_checks_launch(c, (uint32_t)F.pair.size(), F.la.data(), F.lb.data(), F.off.data(),
                                            F.leaves.data(), F.plan, &bad, &first_bad, true);
        if (st != CEC_OK) return st;
        if (bad) {
            c->err = "common cut is not a cut (internal error)";
            return CEC_E_CUT;
        }
        return CEC_OK;
    };
    auto finish_inflight = [&]() -> cec_status {
        cec_status st = collect(inflight);
        if (st != CEC_OK) return st;
        all_v.insert(all_v.end(), inflight.v.begin(), inflight.v.end());
        inflight = Flush();
        return CEC_OK;
    };
    auto flush = [&]() -> cec_status {
        cec_status st = finish_inflight();  // at most one flush in flight
        if (st != CEC_OK) return st;
        std::swap(inflight, buf);
        buf = Flush();
        return launch(inflight);
    };
    std::vector<Cut> common;
    std::vector<std::vector<Cut>> cmn;  // per-pair common cuts of a level computed in parallel
    uint32_t par_min = 2;               // CEC_CUT_PAR_MIN: smallest level run on the pool
    if (const char *e = getenv("CEC_CUT_PAR_MIN")) par_min = std::max(1, atoi(e));
    // CEC_TIMING_LOCAL=1: where a pass spends its host time (stderr)
    static const bool lt = getenv("CEC_TIMING_LOCAL") != nullptr;
    using clk = std::chrono::steady_clock;
    double t_enum = 0, t_common = 0, t_flush = 0;
    auto t_begin = clk::now(), tq = t_begin;
    auto acc = [&](double &a) {
        if (!lt) return;
        const auto t = clk::now();
        a += std::chrono::duration<double, std::milli>(t - tq).count();
        tq = t;
    };
    uint32_t n_par = 0, n_flush = 0, nodes_par = 0, nodes_ser = 0;
    double t_ser = 0;
    // Small cones (<= 64k needed nodes, e.g. C4's 2k): the priority cuts are enumerated without
    // level barriers first — a node starts as soon as its fanins and representative are done (the
    // dependencies of Eq. 2) — and the common cuts of all pairs in parallel; the level loop below
    // then only fills and flushes the buffer, in exactly the level order and at exactly the flush
    // points of Alg. 2, so the checks and verdicts are the same. (Large cones keep the level-by-level
    // loop, whose flushes overlap the enumeration of the next levels.) CEC_ALG2_LEVEL_SYNC=1 forces it.
    size_t n_need = 0;
    for (const auto &L : lists) n_need += L.size();
    const bool dataflow = n_need <= 65536 && getenv("CEC_ALG2_LEVEL_SYNC") == nullptr;
    std::vector<std::vector<Cut>> cmn_all;
    if (dataflow && n_need) {
        if (lt) tq = clk::now();
        std::vector<uint32_t> indeg(N, 0), coff(N + 1, 0), child;
        auto prereq = [&](uint32_t id, uint32_t *out) {  // AND prerequisites of a needed AND node
            int n = 0;
            for (uint32_t p : {c->f0[id] >> 1, c->f1[id] >> 1, repr_of[id]})
                if (p != 0xFFFFFFFFu && p > c->I) out[n++] = p;
            return n;
        };
        uint32_t pq[3];
        for (const auto &L : lists)
            for (uint32_t id : L) {
                const int n = prereq(id, pq);
                indeg[id] = (uint32_t)n;
                for (int t = 0; t < n; ++t) ++coff[pq[t] + 1];
            }
        for (uint32_t i = 0; i < N; ++i) coff[i + 1] += coff[i];
        child.resize(coff[N]);
        {
            std::vector<uint32_t> fillc(coff.begin(), coff.end() - 1);
            for (const auto &L : lists)
                for (uint32_t id : L) {
                    const int n = prereq(id, pq);
                    for (int t = 0; t < n; ++t) child[fillc[pq[t]]++] = id;
                }
        }
        std::mutex mu;
        std::condition_variable cv;
        std::vector<uint32_t> ready;
        size_t remaining = n_need;
        for (const auto &L : lists)
            for (uint32_t id : L)
                if (!indeg[id]) ready.push_back(id);
        pool.run(pool.size() + 1, [&](uint32_t, unsigned) {
            for (;;) {
                uint32_t id;
                {
                    std::unique_lock<std::mutex> l(mu);
                    cv.wait(l, [&]() { return !ready.empty() || remaining == 0; });
                    if (ready.empty()) return;
                    id = ready.back();
                    ready.pop_back();
                }
                node_cuts(J, id, P);
                size_t woke = 0;
                {
                    std::lock_guard<std::mutex> l(mu);
                    --remaining;
                    for (uint32_t t = coff[id]; t < coff[id + 1]; ++t)
                        if (--indeg[child[t]] == 0) ready.push_back(child[t]), ++woke;
                }
                if (woke > 1 || remaining == 0) cv.notify_all();
                else if (woke == 1) cv.notify_one();
            }
        });
        nodes_par = (uint32_t)n_need;
        acc(t_enum);
        cmn_all.resize(npairs);
        pool.run(npairs, [&](uint32_t q, unsigned) { common_cuts_of(P, repr[q], member[q], k_l, max_cuts, cmn_all[q]); });
        acc(t_common);
    }
    for (size_t e = 1; e < lists.size(); ++e) {
        const std::vector<uint32_t> &L = lists[e];
        if (lt) tq = clk::now();
        if (dataflow) {  // cuts and common cuts are ready: Alg. 2 l.11-16 in level order
            for (uint32_t q : pairs_at[e]) {
                const uint32_t la = 2u * repr[q], lb = 2u * member[q] ^ (phase[q] & 1u);
                for (const Cut &x : cmn_all[q]) {
                    buf.pair.push_back(q);
                    buf.la.push_back(la);
                    buf.lb.push_back(lb);
                    buf.leaves.insert(buf.leaves.end(), x.leaf, x.leaf + x.n);
                    buf.off.push_back((uint32_t)buf.leaves.size());
                    log_pair.push_back(q);
                    log_leaves.insert(log_leaves.end(), x.leaf, x.leaf + x.n);
                    log_off.push_back((uint32_t)log_leaves.size());
                    ++nchecks;
                }
            }
            acc(t_common);
            if (buf.pair.size() >= std::max<uint32_t>(1, buffer_checks)) {  // Alg. 2 l.13-14: flush
                ++n_flush;
                cec_status st = flush();
                if (st != CEC_OK) return st;
                acc(t_flush);
            }
            continue;
        }
        // a node's enumeration (~10-25 us at k_l = C = 16) outweighs a pool hand-off, so even
        // levels of 2 nodes run in parallel (C4's carry chains: 109 of 133 levels have < 8 nodes)
        if (L.size() < par_min) {
            for (uint32_t id : L) node_cuts(J, id, P);
            nodes_ser += (uint32_t)L.size();
            acc(t_ser);
        } else {
            ++n_par;
            nodes_par += (uint32_t)L.size();
            pool.run((uint32_t)L.size(), [&](uint32_t i, unsigned) { node_cuts(J, L[i], P); }, true);
            acc(t_enum);
        }
        // Alg. 2 l.11-12: common cuts of the new pairs (in parallel, inserted in pair order)
        const std::vector<uint32_t> &QE = pairs_at[e];
        if (QE.size() >= par_min) {
            if (cmn.size() < QE.size()) cmn.resize(QE.size());
            pool.run((uint32_t)QE.size(), [&](uint32_t i, unsigned) {
                common_cuts_of(P, repr[QE[i]], member[QE[i]], k_l, max_cuts, cmn[i]);
            }, true);
        }
        for (size_t qi = 0; qi < QE.size(); ++qi) {
            const uint32_t q = QE[qi];
            if (QE.size() < par_min) common_cuts_of(P, repr[q], member[q], k_l, max_cuts, common);
            const std::vector<Cut> &cc = QE.size() < par_min ? common : cmn[qi];
            const uint32_t la = 2u * repr[q], lb = 2u * member[q] ^ (phase[q] & 1u);
            for (const Cut &x : cc) {
                buf.pair.push_back(q);
                buf.la.push_back(la);
                buf.lb.push_back(lb);
                buf.leaves.insert(buf.leaves.end(), x.leaf, x.leaf + x.n);
                buf.off.push_back((uint32_t)buf.leaves.size());
                log_pair.push_back(q);
                log_leaves.insert(log_leaves.end(), x.leaf, x.leaf + x.n);
                log_off.push_back((uint32_t)log_leaves.size());
                ++nchecks;
            }
        }
        acc(t_common);
        if (buf.pair.size() >= std::max<uint32_t>(1, buffer_checks)) {  // Alg. 2 l.13-14: flush
            ++n_flush;
            cec_status st = flush();
            if (st != CEC_OK) return st;
            acc(t_flush);
        }
    }
    if (lt) tq = clk::now();
    cec_status st = flush();  // Alg. 2 l.18: the remainder
    if (st == CEC_OK) st = finish_inflight();
    if (st != CEC_OK) return st;
    acc(t_flush);
    if (lt)
        fprintf(stderr, "[cec] local pass %d: %zu levels (%u parallel, %u nodes; serial %u nodes), %u pairs, %u checks, "
                        "%u+1 flushes: enum par %.2f ser %.2f  common %.2f  flush %.2f  total %.2f ms\n", pass_id,
                lists.size(), n_par, nodes_par, nodes_ser, npairs, nchecks, n_flush, t_enum, t_ser, t_common, t_flush,
                std::chrono::duration<double, std::milli>(clk::now() - t_begin).count());
    *num_checks_out = nchecks;
    // optional check log (caller capacities: npairs*max_cuts checks, npairs*max_cuts*k_l leaves)
    if (check_pair) std::memcpy(check_pair, log_pair.data(), 4 * log_pair.size());
    if (check_cut_off) std::memcpy(check_cut_off, log_off.data(), 4 * log_off.size());
    if (check_leaves && !log_leaves.empty()) std::memcpy(check_leaves, log_leaves.data(), 4 * log_leaves.size());
    if (check_verdict && !all_v.empty()) std::memcpy(check_verdict, all_v.data(), 4 * all_v.size());
    return CEC_OK;
}
