// jit.cpp — register-resident window kernels generated per window STRUCTURE and compiled at plan
// time with NVRTC for sm_100a (CEC_ENGINE_JIT / AUTO).
//
// Why: the interpreter keeps node words in shared-memory slots, so every AND costs two loads and a
// store of shared memory (~12 B per node-word) — it is bound by the shared-memory pipe, far below
// the ALU (LOP3) pipe. A window's structure is fixed for the whole 2^k-pattern sweep, so we emit it
// as straight-line code: every node word lives in a register and every AND is exactly ONE
// `lop3.b32` whose 8-bit LUT folds both edge complements (0xC0 = a&b, 0x0C = !a&b, 0x30 = a&!b,
// 0x03 = !a&!b). The LOP3s are emitted as inline PTX so the compiler cannot re-associate or
// simplify the Boolean logic (that would silently skip node evaluations and falsify the
// node-pattern count W; ptxas still allocates registers and schedules). Input (projection) words
// are generated arithmetically from the word index; compares are warp-aggregated
// (__any_sync, __ballot_sync) exactly like the interpreter, so the canonical minimum CEX index is
// the same.
//
// Windows with identical structure (same k, same node list up to renaming, same compares) share
// one compiled kernel; all their instances run in one launch (e.g. the disjoint copies of C5).
#include <cuda_runtime.h>
#include <dlfcn.h>

#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <functional>
#include <map>
#include <memory>
#include <mutex>
#include <string>
#include <vector>

#include "cec_internal.hpp"

namespace cec {

namespace {

// ---- NVRTC, loaded on demand --------------------------------------------------------------------
typedef int nvrtcResult_t;
typedef struct _nvrtcProgram *nvrtcProgram_t;
struct Nvrtc {
    void *h = nullptr;
    nvrtcResult_t (*create)(nvrtcProgram_t *, const char *, const char *, int, const char *const *,
                            const char *const *) = nullptr;
    nvrtcResult_t (*compile)(nvrtcProgram_t, int, const char *const *) = nullptr;
    nvrtcResult_t (*log_size)(nvrtcProgram_t, size_t *) = nullptr;
    nvrtcResult_t (*log)(nvrtcProgram_t, char *) = nullptr;
    nvrtcResult_t (*cubin_size)(nvrtcProgram_t, size_t *) = nullptr;
    nvrtcResult_t (*cubin)(nvrtcProgram_t, char *) = nullptr;
    nvrtcResult_t (*destroy)(nvrtcProgram_t *) = nullptr;
    nvrtcResult_t (*ptx_size)(nvrtcProgram_t, size_t *) = nullptr;
    nvrtcResult_t (*ptx)(nvrtcProgram_t, char *) = nullptr;
    std::string why;
    bool load() {
        if (h) return true;
        const char *cands[] = {"libnvrtc.so.12", "/usr/local/cuda/lib64/libnvrtc.so.12", "libnvrtc.so"};
        for (const char *c : cands) {
            h = dlopen(c, RTLD_NOW | RTLD_LOCAL);
            if (h) break;
        }
        if (!h) {
            why = "libnvrtc.so.12 not found";
            return false;
        }
        create = (decltype(create))dlsym(h, "nvrtcCreateProgram");
        compile = (decltype(compile))dlsym(h, "nvrtcCompileProgram");
        log_size = (decltype(log_size))dlsym(h, "nvrtcGetProgramLogSize");
        log = (decltype(log))dlsym(h, "nvrtcGetProgramLog");
        cubin_size = (decltype(cubin_size))dlsym(h, "nvrtcGetCUBINSize");
        cubin = (decltype(cubin))dlsym(h, "nvrtcGetCUBIN");
        destroy = (decltype(destroy))dlsym(h, "nvrtcDestroyProgram");
        ptx_size = (decltype(ptx_size))dlsym(h, "nvrtcGetPTXSize");
        ptx = (decltype(ptx))dlsym(h, "nvrtcGetPTX");
        if (!(create && compile && log_size && log && cubin_size && cubin && destroy && ptx_size && ptx)) {
            why = "libnvrtc is missing symbols";
            return false;
        }
        return true;
    }
};
Nvrtc g_nvrtc;
std::mutex g_mu;

const char *kMask[5] = {"0xAAAAAAAAu", "0xCCCCCCCCu", "0xF0F0F0F0u", "0xFF00FF00u", "0xFFFF0000u"};

std::string ref_name(const JitProgram &p, uint32_t ref) {
    if (ref == 0) return "0u";
    if (ref <= p.k) return "x" + std::to_string(ref - 1);
    return "n" + std::to_string(ref - p.k - 1);
}

}  // namespace

struct JitKernel {
    cudaLibrary_t lib = nullptr;
    cudaKernel_t kern = nullptr;
    int block = 128;
    int blocks_per_sm = 0;
    int slices_per_pass = 1;  // block-synchronous kernels: warps per block
    bool free_warps = false;  // static per-warp partition: grid fixed at plan time, `ctr` = CSR offsets
    uint32_t lop3 = 0;        // LOP3 instructions per word of the mapped window (structure 0)
    std::vector<uint32_t> lop3s;  // per structure of a bundle (sid order)
    std::vector<uint32_t> imads;  // IMAD cells per word, per structure (mode 3)
    double compile_ms = 0;
    size_t src_bytes = 0, cubin_bytes = 0;
};

std::string jit_key(const JitProgram &p) {
    std::string key;
    key.reserve(16 + 8 * (p.nodes.size() + p.cmps.size()));
    auto put = [&](uint32_t v) { key.append(reinterpret_cast<const char *>(&v), 4); };
    put(p.k);
    put((uint32_t)p.nodes.size());
    put((uint32_t)p.cmps.size());
    for (uint32_t v : p.nodes) put(v);
    for (uint32_t v : p.cmps) put(v);
    return key;
}

// ---- 3-input LUT mapping of the window (one LOP3 per LUT) ----------------------------------------
// An AND node whose only reader is the next AND up (single fanout inside the window, not a compare
// root) need not be materialised: the reader's LOP3 can take the absorbed node's fanins directly,
// as long as the union of leaves stays <= 3 (a LOP3 evaluates ANY 3-input function from an 8-bit
// LUT). Greedy, in topological order: absorb both fanins if possible, else one, else none. Every AND
// node is still evaluated exactly (inside the LUT of its reader); only the register write of the
// absorbed intermediate disappears. The LUT is obtained by evaluating the absorbed expression on
// the canonical truth tables of the LOP3 inputs (a = 0xF0, b = 0xCC, c = 0xAA).
struct MappedNode {
    bool absorbed = false;
    uint8_t nleaves = 0;
    uint32_t leaf[3] = {0, 0, 0};  // operand refs (IMAD: leaf[0] = y, leaf[1] = the word-uniform input m)
    uint8_t tt = 0;                // LOP3 table over the STORED leaf values
    bool imad = false;             // cell on the FMA pipe: mad.lo.u32 (see imad_cell below)
    uint8_t imad_c = 0;            // addend of the mad: 0 = m, 1 = y, 2 = -1
    bool pol = false;              // the register holds the complement of the node's function
};

std::vector<MappedNode> jit_map(const JitProgram &p, bool fuse) {
    const uint32_t n = (uint32_t)(p.nodes.size() / 2), ncmp = (uint32_t)(p.cmps.size() / 2);
    std::vector<uint32_t> uses(p.k + 1 + n, 0);
    for (uint32_t i = 0; i < 2 * n; ++i) ++uses[p.nodes[i] >> 1];
    std::vector<bool> root(p.k + 1 + n, false);
    for (uint32_t i = 0; i < 2 * ncmp; ++i) root[p.cmps[i] >> 1] = true;
    std::vector<MappedNode> m(n);
    auto is_node = [&](uint32_t ref) { return ref > p.k; };
    // value of operand (ref, compl) as an 8-bit truth table over the chosen leaves
    std::function<uint8_t(uint32_t, uint32_t, const MappedNode &, bool)> eval;
    for (uint32_t t = 0; t < n; ++t) {
        const uint32_t oa = p.nodes[2 * t], ob = p.nodes[2 * t + 1];
        const uint32_t ra = oa >> 1, rb = ob >> 1;
        auto can = [&](uint32_t r) {
            return fuse && is_node(r) && uses[r] == 1 && !root[r] && r - p.k - 1 < t;
        };
        auto leaves_of = [&](uint32_t r, bool expand, std::vector<uint32_t> &L) {
            if (expand) {
                const MappedNode &u = m[r - p.k - 1];
                for (int i = 0; i < u.nleaves; ++i) L.push_back(u.leaf[i]);
            } else {
                L.push_back(r);
            }
        };
        MappedNode best;
        bool done = false;
        const bool opts[4][2] = {{true, true}, {true, false}, {false, true}, {false, false}};
        for (auto &o : opts) {
            const bool ea = o[0] && can(ra), eb = o[1] && can(rb);
            if ((o[0] && !ea) || (o[1] && !eb)) continue;
            std::vector<uint32_t> L;
            leaves_of(ra, ea, L);
            leaves_of(rb, eb, L);
            std::sort(L.begin(), L.end());
            L.erase(std::unique(L.begin(), L.end()), L.end());
            if (L.size() > 3) continue;
            MappedNode cand;
            cand.nleaves = (uint8_t)L.size();
            for (size_t i = 0; i < L.size(); ++i) cand.leaf[i] = L[i];
            static const uint8_t K[3] = {0xF0, 0xCC, 0xAA};
            auto leaf_tt = [&](uint32_t r) -> uint8_t {
                for (int i = 0; i < cand.nleaves; ++i)
                    if (cand.leaf[i] == r) return K[i];
                return 0;  // unreachable
            };
            auto operand_tt = [&](uint32_t r, uint32_t c, bool expand) -> uint8_t {
                uint8_t v;
                if (expand) {  // evaluate the absorbed node's own LUT on the new leaf constants
                    const MappedNode &u = m[r - p.k - 1];
                    uint8_t in[3] = {0, 0, 0};
                    for (int i = 0; i < u.nleaves; ++i) in[i] = leaf_tt(u.leaf[i]);
                    v = 0;
                    for (int bit = 0; bit < 8; ++bit) {
                        const int idx = (((in[0] >> bit) & 1) << 2) | (((in[1] >> bit) & 1) << 1) | ((in[2] >> bit) & 1);
                        // u.tt bit for inputs (x0, x1, x2) sits at position 4*x0 + 2*x1 + x2
                        v |= (uint8_t)(((u.tt >> idx) & 1) << bit);
                    }
                } else {
                    v = leaf_tt(r);
                }
                return c ? (uint8_t)~v : v;
            };
            cand.tt = operand_tt(ra, oa & 1u, ea) & operand_tt(rb, ob & 1u, eb);
            best = cand;
            if (ea) m[ra - p.k - 1].absorbed = true;
            if (eb && rb != ra) m[rb - p.k - 1].absorbed = true;
            done = true;
            break;
        }
        (void)done;
        m[t].nleaves = best.nleaves;
        for (int i = 0; i < 3; ++i) m[t].leaf[i] = best.leaf[i];
        m[t].tt = best.tt;
    }
    return m;
}

// ---- area-oriented 3-LUT mapping (fuse mode 2) -----------------------------------------------------
// Every node gets its 3-feasible cuts (merged from its fanins' cuts, like Eq. (1) with k = 3); the
// best cut minimises the area flow AF(n) = 1 + sum_{leaf l} AF(l) / fanout(l) (inputs: 0). Mapping
// then walks from the compare roots down: a node is materialised (one LOP3) iff it is a root or a
// leaf of a chosen cut; every other AND is evaluated inside the LUT of the node that covers it
// (possibly inside several LUTs — duplication is what lets multi-fanout logic be absorbed too).
//
// Dual-pipe cells (mode 3). The ALU pipe that runs LOP3 is the bound (64 LOP3/clk/SM); the FMA pipe
// beside it (IMAD, same rate, B300_MICROARCH.md "Pipe rates") is idle. A window input j >= 5 is
// word-uniform: every u32 word of it is 0 or ~0 (PAPER.md:33 projection words; j = 5..9 depend on
// the lane, j >= 10 on the slice). For such an m and ANY word y, mad.lo.u32 computes exact bitwise
// logic: y*m + m = ~y & m, y*m + y = y & ~m, y*m - 1 = ~(y & m) (m = 0 -> the addend; m = ~0 = -1
// -> addend - y). So a node whose function over a 2-leaf cut {y, m} is an AND of the two with any
// edge complements except ~y & ~m can be evaluated by ONE IMAD on the FMA pipe (the register then
// holds the function or its complement; readers fold that polarity into their LOP3 tables, just as
// they fold edge complements). Every AND node is still evaluated on every pattern — on the other
// pipe. m may also be a node whose support lies inside those inputs (its words are 0 or ~0 too).
// The mapper prices an IMAD cell at `imad_cost` LUTs (the measured ALU cost of its register reads,
// scripts/pipes.cu), so it takes them where they relieve the ALU pipe. ~y & ~m has no form with
// operands y, m, -1; it becomes y & ~m when y's register holds the complement (LOP3 outputs take the
// polarity most of their IMAD readers need), else the cell falls back to a LOP3. XOR-type cuts stay
// LOP3s. jit_verify_map emulates the result against the AIG (CEC_JIT_VERIFY).
namespace {
constexpr uint8_t kLeafTT[3] = {0xF0, 0xCC, 0xAA};
// g = the 2-input function of (y, m) as a 4-bit table, bit (2*y + m). Returns the IMAD form
// (addend: 0 = m, 1 = y, 2 = -1; *pol: register holds the complement) or -1 if none exists.
int imad_cell(uint8_t g, bool *pol) {
    switch (g) {
        case 0x2: *pol = false; return 0;  // ~y & m   = y*m + m
        case 0x4: *pol = false; return 1;  // y & ~m   = y*m + y
        case 0x7: *pol = false; return 2;  // ~(y & m) = y*m - 1
        case 0x8: *pol = true; return 2;   // y & m    = ~(y*m - 1)
        case 0xB: *pol = true; return 1;   // y | ~m   = ~(y*m + y)
        case 0xD: *pol = true; return 0;   // ~y | m   = ~(y*m + m)
        default: return -1;
    }
}
// 4-bit (y, m) table of an 8-bit LOP3-style table whose leaf ypos / mpos carry y / m
uint8_t g_of(uint8_t tt, int ypos, int mpos) {
    uint8_t g = 0;
    for (int yv = 0; yv < 2; ++yv)
        for (int mv = 0; mv < 2; ++mv) {
            int idx = 0;
            idx |= yv << (2 - ypos);
            idx |= mv << (2 - mpos);
            g |= (uint8_t)(((tt >> idx) & 1) << (2 * yv + mv));
        }
    return g;
}
}  // namespace

std::vector<MappedNode> jit_map_area(const JitProgram &p, double imad_cost) {
    const uint32_t n = (uint32_t)(p.nodes.size() / 2), ncmp = (uint32_t)(p.cmps.size() / 2);
    const uint32_t R = p.k + 1 + n;
    struct C3 {
        uint8_t m;
        uint8_t tt;  // the node's function over l[0..m-1] at (0xF0, 0xCC, 0xAA); const-0 leaves read 0
        uint32_t l[3];
    };
    const bool dual = imad_cost >= 0.0;
    // word-uniform signals: inputs j >= 5 and every node whose support lies inside them (its words
    // are then 0 or ~0 too); CEC_MAP_WU_NODES=0 keeps the inputs only
    static const bool wu_nodes = !getenv("CEC_MAP_WU_NODES") || atoi(getenv("CEC_MAP_WU_NODES")) != 0;
    std::vector<uint8_t> wu(R, 0);
    for (uint32_t r = 6; r <= p.k; ++r) wu[r] = 1;
    if (wu_nodes)
        for (uint32_t t = 0; t < n; ++t) {
            const uint32_t a = p.nodes[2 * t] >> 1, b = p.nodes[2 * t + 1] >> 1;
            wu[p.k + 1 + t] = (a == 0 || wu[a]) && (b == 0 || wu[b]);
        }
    auto word_uniform = [&](uint32_t r) { return r != 0 && wu[r] != 0; };
    // an IMAD form for cut c: returns the m leaf position (y = the other) or -1. The form depends
    // on the stored polarities of y and m (see imad_cell); the mapper accepts any AND-type table
    // that has a form now, or could get one by flipping a leaf that is a node (whose polarity is
    // chosen below); the final pass falls back to a LOP3 where no form remains.
    auto imad_pos = [&](const C3 &c) -> int {
        if (!dual || c.m != 2) return -1;
        for (int mp = 1; mp >= 0; --mp) {
            const int yp = 1 - mp;
            if (!word_uniform(c.l[mp]) || c.l[yp] == 0) continue;
            bool pl;
            const uint8_t g = g_of(c.tt, yp, mp);
            if (imad_cell(g, &pl) >= 0) return mp;
            if ((g == 0x1 || g == 0xE) && (c.l[yp] > p.k || c.l[mp] > p.k)) return mp;
        }
        return -1;
    };
    // truth table of cut u re-expressed over the (sorted) leaf list L[0..m)
    auto tt_on = [&](const C3 &u, const uint32_t *L, int m) -> uint8_t {
        uint8_t v[3] = {0, 0, 0};
        for (int i = 0; i < u.m; ++i) {
            if (u.l[i] == 0) continue;
            for (int j = 0; j < m; ++j)
                if (L[j] == u.l[i]) v[i] = kLeafTT[j];
        }
        uint8_t out = 0;
        for (int bit = 0; bit < 8; ++bit) {
            const int idx = (((v[0] >> bit) & 1) << 2) | (((v[1] >> bit) & 1) << 1) | ((v[2] >> bit) & 1);
            out |= (uint8_t)(((u.tt >> idx) & 1) << bit);
        }
        return out;
    };
    std::vector<uint32_t> fanout(R, 0);
    for (uint32_t i = 0; i < 2 * n; ++i) ++fanout[p.nodes[i] >> 1];
    std::vector<bool> root(R, false);
    for (uint32_t i = 0; i < 2 * ncmp; ++i) root[p.cmps[i] >> 1] = true;
    for (uint32_t r = 0; r < R; ++r)
        if (root[r]) ++fanout[r];
    std::vector<std::vector<C3>> cuts(R);
    std::vector<double> af(R, 0.0);
    std::vector<C3> best(R);
    std::vector<uint8_t> bim(R, 0);  // best implementation is an IMAD cell
    std::vector<bool> req(R, false);
    std::vector<double> est(fanout.begin(), fanout.end());  // fanout estimate used by area flow
    static const size_t CAP = getenv("CEC_MAP_CAP") ? (size_t)atoi(getenv("CEC_MAP_CAP")) : 16;
    static const int ITER = getenv("CEC_MAP_ITER") ? atoi(getenv("CEC_MAP_ITER")) : 3;  // area flow, then re-estimate fanouts from the mapping's references
    for (int iter = 0; iter < ITER; ++iter) {
        for (uint32_t r = 0; r < R; ++r) cuts[r].clear();
        for (uint32_t r = 0; r <= p.k; ++r) {
            cuts[r].push_back(C3{1, 0xF0, {r, 0, 0}});
            best[r] = cuts[r][0];
            bim[r] = 0;
            af[r] = 0.0;
        }
        auto cost = [&](const C3 &c) {
            double a = 1.0;
            for (int i = 0; i < c.m; ++i) a += af[c.l[i]] / std::max(1.0, est[c.l[i]]);
            return a;
        };
        for (uint32_t t = 0; t < n; ++t) {
            const uint32_t me = p.k + 1 + t;
            const uint32_t oa = p.nodes[2 * t], ob = p.nodes[2 * t + 1];
            const uint32_t a = oa >> 1, b = ob >> 1;
            std::vector<C3> cand;
            for (const C3 &u : cuts[a])
                for (const C3 &v : cuts[b]) {
                    uint32_t L[6];
                    int m = 0;
                    for (int i = 0; i < u.m; ++i) L[m++] = u.l[i];
                    for (int i = 0; i < v.m; ++i) L[m++] = v.l[i];
                    std::sort(L, L + m);
                    m = (int)(std::unique(L, L + m) - L);
                    if (m > 3) continue;
                    C3 c{(uint8_t)m, 0, {0, 0, 0}};
                    for (int i = 0; i < m; ++i) c.l[i] = L[i];
                    c.tt = (uint8_t)((tt_on(u, L, m) ^ ((oa & 1u) ? 0xFF : 0)) & (tt_on(v, L, m) ^ ((ob & 1u) ? 0xFF : 0)));
                    bool dup = false;
                    for (const C3 &d : cand)
                        if (d.m == c.m && std::equal(d.l, d.l + d.m, c.l)) dup = true;
                    if (!dup) cand.push_back(c);
                }
            std::sort(cand.begin(), cand.end(), [&](const C3 &x, const C3 &y) {
                const double cx = cost(x), cy = cost(y);
                if (cx != cy) return cx < cy;
                if (x.m != y.m) return x.m < y.m;
                return std::lexicographical_compare(x.l, x.l + x.m, y.l, y.l + y.m);
            });
            best[me] = cand[0];  // the trivial {a, b} merge always exists
            af[me] = cost(cand[0]);
            bim[me] = 0;
            for (const C3 &c : cand)  // an IMAD cell over a 2-leaf cut: same flow, cheaper cell
                if (imad_pos(c) >= 0 && cost(c) - 1.0 + imad_cost < af[me]) {
                    best[me] = c;
                    af[me] = cost(c) - 1.0 + imad_cost;
                    bim[me] = 1;
                }
            if (cand.size() > CAP) cand.resize(CAP);
            cuts[me] = cand;
            if (bim[me] && std::find_if(cand.begin(), cand.end(), [&](const C3 &c) {
                    return c.m == best[me].m && std::equal(c.l, c.l + c.m, best[me].l);
                }) == cand.end())
                cuts[me].push_back(best[me]);  // keep the chosen IMAD cut among the node's cuts
            cuts[me].push_back(C3{1, 0xF0, {me, 0, 0}});  // the trivial cut, for readers
        }
        // cover from the roots
        std::fill(req.begin(), req.end(), false);
        std::vector<double> refs(R, 0.0);
        for (uint32_t r = 0; r < R; ++r)
            if (root[r]) {
                req[r] = true;
                refs[r] += 1.0;
            }
        for (uint32_t t = n; t-- > 0;) {
            const uint32_t me = p.k + 1 + t;
            if (!req[me]) continue;
            for (int i = 0; i < best[me].m; ++i) {
                req[best[me].l[i]] = true;
                refs[best[me].l[i]] += 1.0;
            }
        }
        for (uint32_t r = 0; r < R; ++r) est[r] = 0.5 * est[r] + 0.5 * std::max(1.0, refs[r]);
    }
    // exact local area recovery: with the cover's reference counts, each node in topological order
    // takes the cut whose LUTs NOT already shared with the rest of the cover are fewest (the area
    // it adds if referenced = LUTs that become live; dereferencing gives it back). Two passes.
    // areas in quarter-LUTs: a LOP3 cell = 4, an IMAD cell = round(4 * imad_cost)
    const uint32_t WL = 4, WI = dual ? (uint32_t)std::lround(4.0 * std::max(0.0, imad_cost)) : 4;
    std::vector<int32_t> nref(R, 0);
    for (uint32_t r = 0; r < R; ++r)
        if (root[r]) ++nref[r];
    for (uint32_t t = n; t-- > 0;) {
        const uint32_t me = p.k + 1 + t;
        if (nref[me] > 0)
            for (int i = 0; i < best[me].m; ++i) ++nref[best[me].l[i]];
    }
    std::function<uint32_t(uint32_t)> ref_cut = [&](uint32_t r) -> uint32_t {
        uint32_t a = bim[r] ? WI : WL;
        for (int i = 0; i < best[r].m; ++i) {
            const uint32_t l = best[r].l[i];
            if (l > p.k && nref[l]++ == 0) a += ref_cut(l);
        }
        return a;
    };
    std::function<uint32_t(uint32_t)> deref_cut = [&](uint32_t r) -> uint32_t {
        uint32_t a = bim[r] ? WI : WL;
        for (int i = 0; i < best[r].m; ++i) {
            const uint32_t l = best[r].l[i];
            if (l > p.k && --nref[l] == 0) a += deref_cut(l);
        }
        return a;
    };
    static const int EA = getenv("CEC_MAP_EA") ? atoi(getenv("CEC_MAP_EA")) : 2;
    for (int pass = 0; pass < EA; ++pass)
        for (uint32_t t = 0; t < n; ++t) {
            const uint32_t me = p.k + 1 + t;
            const bool mapped = nref[me] > 0;
            if (mapped) deref_cut(me);
            C3 keep = best[me];
            uint8_t keep_im = bim[me];
            uint32_t best_a = UINT32_MAX;
            for (const C3 &c : cuts[me]) {
                if (c.m == 1 && c.l[0] == me) continue;  // the trivial cut
                for (uint8_t im = 0; im < 2; ++im) {
                    if (im && imad_pos(c) < 0) continue;
                    best[me] = c;
                    bim[me] = im;
                    const uint32_t a = ref_cut(me);
                    deref_cut(me);
                    if (a < best_a) {
                        best_a = a;
                        keep = c;
                        keep_im = im;
                    }
                }
            }
            best[me] = keep;
            bim[me] = keep_im;
            if (mapped) ref_cut(me);
        }
    for (uint32_t r = 0; r < R; ++r) req[r] = nref[r] > 0;
    // LUT truth tables: evaluate the cone between the leaves and the node on (0xF0, 0xCC, 0xAA)
    std::vector<MappedNode> out(n);
    std::vector<uint8_t> val(R, 0);
    std::vector<uint32_t> stamp(R, 0);
    uint32_t ep = 0;
    static const uint8_t K[3] = {0xF0, 0xCC, 0xAA};
    std::function<uint8_t(uint32_t)> ev = [&](uint32_t r) -> uint8_t {
        if (stamp[r] == ep) return val[r];
        uint8_t v;
        if (r == 0) {
            v = 0;
        } else if (r <= p.k) {
            v = 0;  // unreachable for a valid cut (inputs are always leaves)
        } else {
            const uint32_t t = r - p.k - 1;
            const uint32_t oa = p.nodes[2 * t], ob = p.nodes[2 * t + 1];
            const uint8_t va = ev(oa >> 1) ^ (uint8_t)((oa & 1u) ? 0xFF : 0), vb = ev(ob >> 1) ^ (uint8_t)((ob & 1u) ? 0xFF : 0);
            v = va & vb;
        }
        stamp[r] = ep;
        val[r] = v;
        return v;
    };
    // polarity of every materialised signal: the register holds function ^ pol (inputs: 0). A LOP3
    // cell may hold either polarity for free: in topological order it takes the one under which
    // more of its IMAD readers have a form (each reader's other leaf at its polarity if already
    // decided, else as is). An IMAD cell's polarity is fixed by its form.
    std::vector<std::vector<uint32_t>> readers(R);
    for (uint32_t t = 0; t < n; ++t) {
        const uint32_t me = p.k + 1 + t;
        if (req[me] && bim[me] && best[me].m == 2)
            for (int i = 0; i < 2; ++i) readers[best[me].l[i]].push_back(me);
    }
    std::vector<uint8_t> pol(R, 0), decided(R, 0);
    auto flip = [](uint8_t g, bool fy, bool fm) {  // (y, m) table with y and/or m complemented
        uint8_t o = 0;
        for (int yv = 0; yv < 2; ++yv)
            for (int mv = 0; mv < 2; ++mv)
                o |= (uint8_t)(((g >> (2 * yv + mv)) & 1) << (2 * (yv ^ (int)fy) + (mv ^ (int)fm)));
        return o;
    };
    auto reader_fits = [&](uint32_t q, uint32_t who, bool who_pol) {
        const C3 &c = best[q];
        for (int mp = 1; mp >= 0; --mp) {
            const int yp = 1 - mp;
            if (!word_uniform(c.l[mp]) || c.l[yp] == 0) continue;
            auto pl = [&](uint32_t r) { return r == who ? who_pol : (decided[r] ? pol[r] != 0 : false); };
            bool f;
            if (imad_cell(flip(g_of(c.tt, yp, mp), pl(c.l[yp]), pl(c.l[mp])), &f) >= 0) return true;
        }
        return false;
    };
    for (uint32_t t = 0; t < n; ++t) {
        const uint32_t me = p.k + 1 + t;
        MappedNode &x = out[t];
        x.absorbed = !req[me];
        if (x.absorbed) continue;
        const C3 &c = best[me];
        ++ep;
        for (int i = 0; i < c.m; ++i) {  // leaf i is read as its STORED value (polarity folded in)
            stamp[c.l[i]] = ep;
            val[c.l[i]] = c.l[i] == 0 ? 0 : (uint8_t)(K[i] ^ (pol[c.l[i]] ? 0xFF : 0));
        }
        // evaluate node me itself over its cut (its own value is not a leaf)
        const uint32_t oa = p.nodes[2 * t], ob = p.nodes[2 * t + 1];
        const uint8_t va = ev(oa >> 1) ^ (uint8_t)((oa & 1u) ? 0xFF : 0), vb = ev(ob >> 1) ^ (uint8_t)((ob & 1u) ? 0xFF : 0);
        x.tt = va & vb;
        x.nleaves = c.m;
        for (int i = 0; i < 3; ++i) x.leaf[i] = i < c.m ? c.l[i] : 0;
        if (!bim[me] && !readers[me].empty()) {
            int score = 0;
            for (uint32_t q : readers[me]) score += (int)reader_fits(q, me, true) - (int)reader_fits(q, me, false);
            if (score > 0) {  // LOP3 cell holding the complement
                x.tt = (uint8_t)~x.tt;
                x.pol = true;
            }
        }
        if (bim[me]) {  // IMAD cell, if the stored polarity of y still admits a form (else a LOP3)
            for (int mp = 1; mp >= 0 && !x.imad; --mp) {
                const int yp = 1 - mp;
                if (!word_uniform(c.l[mp]) || c.l[yp] == 0) continue;
                bool pl = false;
                const int form = imad_cell(g_of(x.tt, yp, mp), &pl);
                if (form < 0) continue;
                x.imad = true;
                x.imad_c = (uint8_t)form;
                x.pol = pl;
                x.leaf[0] = c.l[yp];
                x.leaf[1] = c.l[mp];
                x.leaf[2] = 0;
            }
        }
        pol[me] = x.pol;
        decided[me] = 1;
    }
    return out;
}

// IMAD cells (mode 3) are emitted by the PTX-splice body only; other code paths map with mode 2
int jit_eff_mode(const JitConfig &cfg) {
    return cfg.fuse == 3 && !(cfg.splice && (cfg.sync_every > 0 || cfg.free_warps)) ? 2 : cfg.fuse;
}

double jit_imad_cost() {  // CEC_MAP_IMAD: price of an IMAD cell in LUTs (mode 3)
    static const double v = getenv("CEC_MAP_IMAD") ? atof(getenv("CEC_MAP_IMAD")) : 0.5;
    return v;
}

std::vector<MappedNode> jit_map_mode(const JitProgram &p, int mode) {
    if (mode == 3) return jit_map_area(p, jit_imad_cost());
    return mode == 2 ? jit_map_area(p, -1.0) : jit_map(p, mode != 0);
}

// Host-side check of a mapping (CEC_JIT_VERIFY=1, and the CPU tests): evaluate the mapped cell
// network exactly as the body executes it (lop3.b32 tables over stored leaf values, mad.lo.u32 with
// 32-bit wrap-around, %cz for missing leaves) on `words` u32 words — inputs 0..4 the P:33 masks,
// inputs >= 5 random 0 / ~0 words (word-uniform, as in the kernels) — and compare every
// materialised cell with the AIG's own AND evaluation, polarity included, and every compare's diff.
const char *jit_verify_map(const JitProgram &p, int mode, uint32_t words, uint64_t seed) {
    static const uint32_t masks[5] = {0xAAAAAAAAu, 0xCCCCCCCCu, 0xF0F0F0F0u, 0xFF00FF00u, 0xFFFF0000u};
    const uint32_t n = (uint32_t)(p.nodes.size() / 2), ncmp = (uint32_t)(p.cmps.size() / 2);
    const std::vector<MappedNode> map = jit_map_mode(p, mode);
    std::vector<uint32_t> v(p.k + 1 + n), st(p.k + 1 + n);
    uint64_t x = seed * 0x9E3779B97F4A7C15ull + 1;
    auto rnd = [&]() {  // splitmix64
        uint64_t z = (x += 0x9E3779B97F4A7C15ull);
        z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
        z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
        return z ^ (z >> 31);
    };
    static thread_local std::string msg;
    // test hook (tests/test_jit_map.py): emulate the first IMAD cell with a wrong addend, so the
    // check itself is shown to catch a wrong cell
    const bool break_imad = getenv("CEC_JIT_BREAK_IMAD") != nullptr;
    uint32_t first_imad = UINT32_MAX;
    for (uint32_t t = 0; t < n && first_imad == UINT32_MAX; ++t)
        if (map[t].imad) first_imad = t;
    for (uint32_t w = 0; w < words; ++w) {
        v[0] = st[0] = 0;
        for (uint32_t j = 0; j < p.k; ++j) v[j + 1] = st[j + 1] = j < 5 ? masks[j] : ((rnd() & 1) ? ~0u : 0u);
        for (uint32_t t = 0; t < n; ++t) {
            const uint32_t oa = p.nodes[2 * t], ob = p.nodes[2 * t + 1], me = p.k + 1 + t;
            v[me] = (v[oa >> 1] ^ ((oa & 1u) ? ~0u : 0u)) & (v[ob >> 1] ^ ((ob & 1u) ? ~0u : 0u));
            const MappedNode &c = map[t];
            if (c.absorbed) continue;
            uint32_t r;
            if (c.imad) {
                const uint32_t y = st[c.leaf[0]], m = st[c.leaf[1]];
                const uint8_t form = (break_imad && t == first_imad) ? (uint8_t)((c.imad_c + 1) % 3) : c.imad_c;
                r = y * m + (form == 0 ? m : form == 1 ? y : ~0u);
            } else {
                const uint32_t a = c.nleaves > 0 ? st[c.leaf[0]] : 0u, b = c.nleaves > 1 ? st[c.leaf[1]] : 0u,
                               d = c.nleaves > 2 ? st[c.leaf[2]] : 0u;
                r = 0;
                for (int bit = 0; bit < 32; ++bit) {
                    const int idx = (((a >> bit) & 1) << 2) | (((b >> bit) & 1) << 1) | ((d >> bit) & 1);
                    r |= (uint32_t)((c.tt >> idx) & 1) << bit;
                }
            }
            st[me] = r;
            if (r != (v[me] ^ (c.pol ? ~0u : 0u))) {
                char b[200];
                snprintf(b, sizeof b, "mapped cell of node %u (%s, pol %d) = %08x, AIG gives %08x", t,
                         c.imad ? "imad" : "lop3", (int)c.pol, r, v[me]);
                msg = b;
                return msg.c_str();
            }
        }
        for (uint32_t q = 0; q < ncmp; ++q) {  // the body's diff: stored a ^ stored b ^ folded polarity
            const uint32_t a = p.cmps[2 * q], b = p.cmps[2 * q + 1];
            auto pl = [&](uint32_t r) { return r > p.k ? map[r - p.k - 1].pol : false; };
            const bool inv = (((a ^ b) & 1u) != 0) != (pl(a >> 1) != pl(b >> 1));
            const uint32_t d = st[a >> 1] ^ st[b >> 1] ^ (inv ? ~0u : 0u);
            const uint32_t want = (v[a >> 1] ^ ((a & 1u) ? ~0u : 0u)) ^ (v[b >> 1] ^ ((b & 1u) ? ~0u : 0u));
            if (d != want) {
                msg = "compare " + std::to_string(q) + ": mapped diff differs from the AIG's";
                return msg.c_str();
            }
        }
    }
    return nullptr;
}

uint32_t jit_lop3_count(const JitProgram &p, int mode, uint32_t *imads) {
    uint32_t c = 0, im = 0;
    for (const MappedNode &x : jit_map_mode(p, mode)) {
        c += !x.absorbed && !x.imad;
        im += x.imad;
    }
    if (imads) *imads = im;
    return c;
}

// Block-synchronous item loop with the NEXT item prefetched behind the current item's body: the
// work-queue atomic and the 16-byte item load are issued at the start of an item (cp.async into the
// other shared slot) and waited for only before the end-of-item barrier, so a block never stalls on
// them (for small windows an item is one pass of ~4 us; a blocking fetch cost ~1.5 us of it).
#define ITEM_PIPELINE                                                                                  \
    "  __shared__ u32 s_it[2]; __shared__ __align__(16) JItem s_item[2];\n"                            \
    "  u32 nxt = 0u;\n"                                                                                \
    "  if (threadIdx.x == 0u) { const u32 t = atomicAdd(ctr, 1u); s_it[0] = t; if (t < nitems) s_item[0] = items[t];\n" \
    "    nxt = atomicAdd(ctr, 1u); }\n"                                                                \
    "  __syncthreads();\n"                                                                            \
    "  for (u32 cur = 0u;; cur ^= 1u) {\n"                                                            \
    "    const u32 it = s_it[cur];\n"                                                                 \
    "    if (it >= nitems) return;\n"
#define ITEM_PREFETCH                                                                                  \
    "    if (threadIdx.x == 0u) {\n"                                                                  \
    "      s_it[cur ^ 1u] = nxt;\n"                                                                   \
    "      if (nxt < nitems) asm volatile(\"cp.async.ca.shared.global [%0], [%1], 16;\" :: \"r\"((u32)__cvta_generic_to_shared(&s_item[cur ^ 1u])), \"l\"(items + nxt) : \"memory\");\n" \
    "      nxt = atomicAdd(ctr, 1u);\n"                                                               \
    "    }\n"
#define ITEM_WAIT "    if (threadIdx.x == 0u) asm volatile(\"cp.async.wait_all;\" ::: \"memory\");\n"

std::string jit_source(const JitProgram &p, const JitConfig &cfg) {
    const uint32_t n = (uint32_t)(p.nodes.size() / 2), ncmp = (uint32_t)(p.cmps.size() / 2);
    // free warps (small bodies, splice only): every warp runs its own static, contiguous share of
    // the group's slices (host-partitioned items, CSR offsets passed in `ctr`): no work-queue
    // atomics and no block barriers at all; the code path below is the block-synchronous one with
    // its loop header and tail replaced
    const bool free_w = cfg.free_warps && cfg.splice;
    // ILP 2 (free warps only): each pass evaluates slices s and s + 1 with two copies of the body
    // (BODY0, BODY1) in one basic block, so ptxas can interleave two independent dependency chains;
    // slice s + 1 past the item's end is computed but its compares are masked (liveB)
    const bool ilp2 = free_w && cfg.ilp == 2;
    const bool block_sync = cfg.sync_every > 0 || free_w;
    const int nw = cfg.threads / 32;
    std::string s;
    s.reserve(96 * (size_t)n + 160 * (size_t)ncmp + 4096);
    char buf[1024];
    s += "typedef unsigned int u32; typedef unsigned long long u64;\n"
         "struct JItem { u32 win, s_begin, s_end, cmp_off; };\n"
         "__device__ __noinline__ void rep(u32 d, u32 c, u32 win, u32 s, u32 lane, u32 ncmp, u32 cmp_off,\n"
         "    u64 *first, u64 *bound, u32 *neq_cnt) {\n"
         "  const u32 bal = __ballot_sync(0xFFFFFFFFu, d != 0u);\n"
         "  const u32 l = (u32)__ffs(bal) - 1u;\n"
         "  const u32 dl = __shfl_sync(0xFFFFFFFFu, d, l);\n"
         "  if (lane != 0u) return;\n"
         "  const u64 idx = ((((u64)s << 5) + l) << 5) + (u32)(__ffs(dl) - 1);\n"
         "  const u64 old = atomicMin_system(&first[cmp_off + c], idx);  /* system scope: peer mode */\n"
         "  if (old != ~0ull) return;\n"
         "  __threadfence_system();\n"
         "  if (atomicAdd_system(&neq_cnt[win], 1u) + 1u != ncmp) return;\n"
         "  __threadfence_system();\n"
         "  u64 mx = 0;\n"
         "  for (u32 t = 0; t < ncmp; ++t) { u64 v = atomicAdd_system(&first[cmp_off + t], 0ull); mx = v > mx ? v : mx; }\n"
         "  atomicMin_system(&bound[win], mx);\n"
         "}\n";
    snprintf(buf, sizeof buf,
             "extern \"C\" __global__ void __launch_bounds__(%d, %d) cecjit(const JItem *__restrict__ items, u32 nitems,\n"
             "    u32 *ctr, u64 *first, u64 *bound, u32 *neq_cnt) {\n"
             "  const u32 lane = threadIdx.x & 31u;\n",
             cfg.threads, cfg.min_blocks);
    s += buf;
    // input (projection) words: word index = 32 s + lane, so inputs 5..9 depend on the
    // lane only (computed once per thread) and inputs >= 10 on the slice only (warp-uniform)
    for (uint32_t j = 5; j < std::min<uint32_t>(p.k, 10); ++j) {
        snprintf(buf, sizeof buf, "  const u32 x%u = 0u - ((lane >> %u) & 1u);\n", j, j - 5);
        s += buf;
    }
    if (free_w) {
        snprintf(buf, sizeof buf,
                 "  const u32 gw = blockIdx.x * %du + (threadIdx.x >> 5);\n"
                 "  const u32 i1 = ctr[gw + 1u];\n"
                 "  for (u32 i = ctr[gw]; i < i1; ++i) {\n"
                 "    const JItem I = items[i];\n"
                 "    u64 bnd = ~0ull;\n"
                 "    for (u32 s = I.s_begin; s < I.s_end; s += %du) {\n"
                 "      if (((u64)s << 10) >= bnd) break;  /* warp-uniform (lane 0's bound, shuffled) */\n"
                 "      const bool live = true;\n"
                 "      u64 bnd_next = 0ull;\n"
                 "      if (lane == 0u) bnd_next = *((volatile u64 *)&bound[I.win]);  // used next slice\n",
                 nw, ilp2 ? 2 : 1);
        s += buf;
    } else if (!block_sync) {
        // every warp independent: pulls items itself, one 32-word slice per pass
        s += "  for (;;) {\n"
             "    u32 it = 0;\n"
             "    if (lane == 0u) it = atomicAdd(ctr, 1u);\n"
             "    it = __shfl_sync(0xFFFFFFFFu, it, 0);\n"
             "    if (it >= nitems) return;\n"
             "    const JItem I = items[it];\n"
             "    for (u32 s = I.s_begin; s < I.s_end; ++s) {\n"
             "      u64 bw = 0ull;\n"
             "      if (lane == 0u) bw = *((volatile u64 *)&bound[I.win]);\n"
             "      if (((u64)s << 10) >= __shfl_sync(0xFFFFFFFFu, bw, 0)) break;  /* warp-uniform exit */\n"
             "      const bool live = true;\n";
    } else {
        // block-synchronous: the block pulls an item and its warps take consecutive slices; a
        // __syncthreads() every few hundred nodes keeps all warps of the SM inside the same stretch
        // of the (large, straight-line) program so instruction-cache lines are shared, not thrashed
        s += "  const u32 warp = threadIdx.x >> 5;\n" ITEM_PIPELINE "    const JItem I = s_item[cur];\n" ITEM_PREFETCH;
        snprintf(buf, sizeof buf,
                 "    u64 bnd = ~0ull;  /* first pass of an item: no skip test, so no exposed bound load */\n"
                 "    for (u32 s0 = I.s_begin; s0 < I.s_end; s0 += %du) {\n"
                 "      const u32 s = s0 + warp;\n"
                 "      const bool live = s < I.s_end && ((u64)s << 10) < bnd;\n"
                 "      if (!__syncthreads_or(live)) break;\n"
                 "      const u64 bnd_next = *((volatile u64 *)&bound[I.win]);  // used next pass: latency hidden\n",
                 nw);
        s += buf;
    }
    for (uint32_t j = 0; j < p.k; ++j) {
        if (j < 5)
            snprintf(buf, sizeof buf, "      const u32 x%u = %s;\n", j, kMask[j]);
        else if (j < 10)
            continue;  // lane-only, hoisted above
        else
            snprintf(buf, sizeof buf, "      const u32 x%u = 0u - ((s >> %u) & 1u);\n", j, j - 10);
        s += buf;
    }
    if (ilp2) {
        s += "      const u32 sB = s + 1u;\n      const bool liveB = sB < I.s_end;\n";
        for (uint32_t j = 0; j < p.k; ++j) {
            if (j < 10)
                snprintf(buf, sizeof buf, "      const u32 y%u = x%u;\n", j, j);
            else
                snprintf(buf, sizeof buf, "      const u32 y%u = 0u - ((sB >> %u) & 1u);\n", j, j - 10);
            s += buf;
        }
    }
    // compares are placed right after their later root so roots die early (fewer live registers)
    std::vector<std::vector<uint32_t>> after(n + 1);
    for (uint32_t c = 0; c < ncmp; ++c) {
        const uint32_t ra = p.cmps[2 * c] >> 1, rb = p.cmps[2 * c + 1] >> 1;
        const uint32_t m = std::max(ra, rb);
        after[m > p.k ? m - p.k : 0].push_back(c);
    }
    auto emit_cmp = [&](uint32_t c) {
        const uint32_t a = p.cmps[2 * c], b = p.cmps[2 * c + 1];
        const bool inv = ((a ^ b) & 1u) != 0;
        snprintf(buf, sizeof buf,
                 "      { const u32 d = live ? (%s%s ^ %s%s) : 0u; if (__any_sync(0xFFFFFFFFu, d != 0u)) rep(d, %uu, I.win, s, lane, %uu, I.cmp_off, first, bound, neq_cnt); }\n",
                 inv ? "~(" : "", ref_name(p, a >> 1).c_str(), ref_name(p, b >> 1).c_str(), inv ? ")" : "", c, ncmp);
        s += buf;
    };
    if (cfg.splice && block_sync) {
        // PTX-splice mode: the whole LUT network is ONE inline-asm statement whose text is a marker
        // with its operands; the body PTX is generated directly and spliced in after NVRTC
        // (jit_body_ptx), so NVVM never sees the thousands of LUTs. Compares inside the body vote
        // per warp; a mismatching compare sets its bit in the warp masks m* and stores the lanes'
        // diff words to dbuf (rare path), so only the masks stay live through the body.
        const uint32_t M = (ncmp + 31) / 32;
        // body b: masks m<b>_*, diff buffer dbuf<b>, inputs x* (b = 0) or y* (b = 1, ILP 2)
        const int nb = ilp2 ? 2 : 1;
        for (int b = 0; b < nb; ++b) {
            if (ncmp) {
                snprintf(buf, sizeof buf, "      u32 dbuf%d[%u];\n", b, ncmp);
                s += buf;
            }
            for (uint32_t w = 0; w < M; ++w) {
                snprintf(buf, sizeof buf, "      u32 m%d_%u;\n", b, w);
                s += buf;
            }
        }
        for (int b = 0; b < nb; ++b) {
            snprintf(buf, sizeof buf, "      asm volatile(\"//@@BODY%d@@", b);
            s += buf;
            for (uint32_t i = 0; i < M + p.k + (ncmp ? 1 : 0); ++i) {
                snprintf(buf, sizeof buf, " %%%u", i);
                s += buf;
            }
            s += "\" :";
            for (uint32_t w = 0; w < M; ++w) {
                snprintf(buf, sizeof buf, "%s \"=r\"(m%d_%u)", w ? "," : "", b, w);
                s += buf;
            }
            s += " :";
            for (uint32_t j = 0; j < p.k; ++j) {
                snprintf(buf, sizeof buf, "%s \"r\"(%c%u)", j ? "," : "", b ? 'y' : 'x', j);
                s += buf;
            }
            if (ncmp) {
                snprintf(buf, sizeof buf, ", \"l\"(dbuf%d)", b);
                s += buf;
            }
            s += " : \"memory\");\n";
        }
        for (int b = 0; b < nb; ++b)
            for (uint32_t w = 0; w < M; ++w) {
                snprintf(buf, sizeof buf,
                         "      for (u32 mk = m%d_%u; mk; mk &= mk - 1u) { const u32 c = %uu + (u32)__ffs(mk) - 1u;\n"
                         "        const u32 d = %s ? dbuf%d[c] : 0u;\n"
                         "        if (__any_sync(0xFFFFFFFFu, d != 0u)) rep(d, c, I.win, %s, lane, %uu, I.cmp_off, first, bound, neq_cnt); }\n",
                         b, w, 32 * w, b ? "liveB" : "live", b, b ? "sB" : "s", ncmp);
                s += buf;
            }
    } else {
        const std::vector<MappedNode> map = jit_map_mode(p, jit_eff_mode(cfg));
        uint32_t lut_total = 0;
        for (const MappedNode &x : map) lut_total += !x.absorbed;
        for (uint32_t c : after[0]) emit_cmp(c);
        uint32_t emitted = 0;
        for (uint32_t t = 0; t < n; ++t) {
            const MappedNode &x = map[t];
            if (!x.absorbed) {
                // LOP3 input order (a, b, c) = leaf[0..2]; the LUT was built for (0xF0, 0xCC, 0xAA)
                snprintf(buf, sizeof buf,
                         "      u32 n%u; asm(\"lop3.b32 %%0, %%1, %%2, %%3, 0x%02X;\" : \"=r\"(n%u) : \"r\"(%s), \"r\"(%s), \"r\"(%s));\n",
                         t, x.tt, t, x.nleaves > 0 ? ref_name(p, x.leaf[0]).c_str() : "0u",
                         x.nleaves > 1 ? ref_name(p, x.leaf[1]).c_str() : "0u",
                         x.nleaves > 2 ? ref_name(p, x.leaf[2]).c_str() : "0u");
                s += buf;
                ++emitted;
            }
            for (uint32_t c : after[t + 1]) emit_cmp(c);
            // keep the block's warps in one stretch of a large body (shared I-cache lines); a small body
            // (<= 2048 LUTs, <= 32 KB of SASS) fits the caches and needs no mid-body barrier
            if (block_sync && !x.absorbed && lut_total > 2048 && emitted % (uint32_t)cfg.sync_every == 0)
                s += "      __syncthreads();\n";
        }
    }
    if (free_w)
        s += "      bnd = __shfl_sync(0xFFFFFFFFu, bnd_next, 0);\n    }\n  }\n}\n";
    else
        s += block_sync ? "      bnd = __shfl_sync(0xFFFFFFFFu, bnd_next, 0);\n    }\n" ITEM_WAIT "    __syncthreads();\n  }\n}\n" : "    }\n  }\n}\n";
    return s;
}

// Bundle kernel: several window STRUCTURES in one kernel (splice + block-synchronous mode only).
// Items carry (window | sid << 20); the block takes an item, every warp computes the input words
// of its slice once and the item's structure body runs from a switch. Used for structures whose own
// launch could not fill the GPU (single small windows, e.g. most of C3's): one persistent grid pulls
// the items of all of them, instead of hundreds of tiny launches serialised over a few streams.
std::string jit_source_bundle(const std::vector<const JitProgram *> &ps, const JitConfig &cfg) {
    const int nw = cfg.threads / 32;
    uint32_t kmax = 0;
    for (const JitProgram *p : ps) kmax = std::max(kmax, p->k);
    std::string s;
    char buf[1024];
    s += "typedef unsigned int u32; typedef unsigned long long u64;\n"
         "struct JItem { u32 win, s_begin, s_end, cmp_off; };\n"
         "__device__ __noinline__ void rep(u32 d, u32 c, u32 win, u32 s, u32 lane, u32 ncmp, u32 cmp_off,\n"
         "    u64 *first, u64 *bound, u32 *neq_cnt) {\n"
         "  const u32 bal = __ballot_sync(0xFFFFFFFFu, d != 0u);\n"
         "  const u32 l = (u32)__ffs(bal) - 1u;\n"
         "  const u32 dl = __shfl_sync(0xFFFFFFFFu, d, l);\n"
         "  if (lane != 0u) return;\n"
         "  const u64 idx = ((((u64)s << 5) + l) << 5) + (u32)(__ffs(dl) - 1);\n"
         "  const u64 old = atomicMin_system(&first[cmp_off + c], idx);  /* system scope: peer mode */\n"
         "  if (old != ~0ull) return;\n"
         "  __threadfence_system();\n"
         "  if (atomicAdd_system(&neq_cnt[win], 1u) + 1u != ncmp) return;\n"
         "  __threadfence_system();\n"
         "  u64 mx = 0;\n"
         "  for (u32 t = 0; t < ncmp; ++t) { u64 v = atomicAdd_system(&first[cmp_off + t], 0ull); mx = v > mx ? v : mx; }\n"
         "  atomicMin_system(&bound[win], mx);\n"
         "}\n";
    snprintf(buf, sizeof buf,
             "extern \"C\" __global__ void __launch_bounds__(%d, %d) cecjit(const JItem *__restrict__ items, u32 nitems,\n"
             "    u32 *ctr, u64 *first, u64 *bound, u32 *neq_cnt) {\n",
             cfg.threads, cfg.min_blocks);
    s += buf;
    const bool free_w = cfg.free_warps;
    if (free_w) {  // static per-warp partition (see jit_source): items = (window | sid << 20, slices)
        snprintf(buf, sizeof buf,
                 "  const u32 lane = threadIdx.x & 31u;\n"
                 "  const u32 gw = blockIdx.x * %du + (threadIdx.x >> 5);\n"
                 "  const u32 i1 = ctr[gw + 1u];\n"
                 "  for (u32 i = ctr[gw]; i < i1; ++i) {\n"
                 "    JItem I = items[i];\n"
                 "    const u32 sid = I.win >> 20;\n"
                 "    I.win &= 0xFFFFFu;\n"
                 "    u64 bnd = ~0ull;\n"
                 "    for (u32 s = I.s_begin; s < I.s_end; ++s) {\n"
                 "      if (((u64)s << 10) >= bnd) break;\n"
                 "      const bool live = true;\n"
                 "      u64 bnd_next = 0ull;\n"
                 "      if (lane == 0u) bnd_next = *((volatile u64 *)&bound[I.win]);\n",
                 nw);
        s += buf;
    } else {
        s += "  const u32 lane = threadIdx.x & 31u;\n"
             "  const u32 warp = threadIdx.x >> 5;\n" ITEM_PIPELINE "    JItem I = s_item[cur];\n" ITEM_PREFETCH;
        snprintf(buf, sizeof buf,
                 "    const u32 sid = I.win >> 20;\n"
                 "    I.win &= 0xFFFFFu;\n"
                 "    u64 bnd = ~0ull;  /* first pass of an item: no skip test, so no exposed bound load */\n"
                 "    for (u32 s0 = I.s_begin; s0 < I.s_end; s0 += %du) {\n"
                 "      const u32 s = s0 + warp;\n"
                 "      const bool live = s < I.s_end && ((u64)s << 10) < bnd;\n"
                 "      if (!__syncthreads_or(live)) break;\n"
                 "      const u64 bnd_next = *((volatile u64 *)&bound[I.win]);\n",
                 nw);
        s += buf;
    }
    for (uint32_t j = 0; j < kmax; ++j) {
        if (j < 5)
            snprintf(buf, sizeof buf, "      const u32 x%u = %s;\n", j, kMask[j]);
        else if (j < 10)
            snprintf(buf, sizeof buf, "      const u32 x%u = 0u - ((lane >> %u) & 1u);\n", j, j - 5);
        else
            snprintf(buf, sizeof buf, "      const u32 x%u = 0u - ((s >> %u) & 1u);\n", j, j - 10);
        s += buf;
    }
    s += "      switch (sid) {\n";
    for (size_t i = 0; i < ps.size(); ++i) {
        const JitProgram &p = *ps[i];
        const uint32_t ncmp = (uint32_t)(p.cmps.size() / 2), M = (ncmp + 31) / 32;
        snprintf(buf, sizeof buf, "      case %zuu: {\n", i);
        s += buf;
        if (ncmp) {
            snprintf(buf, sizeof buf, "        u32 dbuf[%u];\n", ncmp);
            s += buf;
        }
        for (uint32_t w = 0; w < M; ++w) {
            snprintf(buf, sizeof buf, "        u32 m%u;\n", w);
            s += buf;
        }
        snprintf(buf, sizeof buf, "        asm volatile(\"//@@BODY%zu@@", i);
        s += buf;
        for (uint32_t t = 0; t < M + p.k + (ncmp ? 1 : 0); ++t) {
            snprintf(buf, sizeof buf, " %%%u", t);
            s += buf;
        }
        s += "\" :";
        for (uint32_t w = 0; w < M; ++w) {
            snprintf(buf, sizeof buf, "%s \"=r\"(m%u)", w ? "," : "", w);
            s += buf;
        }
        s += " :";
        for (uint32_t j = 0; j < p.k; ++j) {
            snprintf(buf, sizeof buf, "%s \"r\"(x%u)", j ? "," : "", j);
            s += buf;
        }
        if (ncmp) s += ", \"l\"(dbuf)";
        s += " : \"memory\");\n";
        for (uint32_t w = 0; w < M; ++w) {
            snprintf(buf, sizeof buf,
                     "        for (u32 mk = m%u; mk; mk &= mk - 1u) { const u32 c = %uu + (u32)__ffs(mk) - 1u;\n"
                     "          const u32 d = live ? dbuf[c] : 0u;\n"
                     "          if (__any_sync(0xFFFFFFFFu, d != 0u)) rep(d, c, I.win, s, lane, %uu, I.cmp_off, first, bound, neq_cnt); }\n",
                     w, 32 * w, ncmp);
            s += buf;
        }
        s += "      } break;\n";
    }
    s += "      default: break;\n      }\n      bnd = __shfl_sync(0xFFFFFFFFu, bnd_next, 0);\n    }\n";
    s += free_w ? "  }\n}\n" : ITEM_WAIT "    __syncthreads();\n  }\n}\n";
    return s;
}

// PTX of the LUT network for splice mode: out_regs[c] receive the compare diffs, in_regs[j] hold
// the input words. One lop3.b32 per materialised LUT (mapping of jit_map_mode), a bar.sync every
// sync_every LUTs for large bodies, and d_c = a ^ b (^ ~0) right after the later root.
std::string jit_body_ptx(const JitProgram &p, const JitConfig &cfg, const std::vector<std::string> &masks,
                         const std::vector<std::string> &in_regs, const std::string &dbuf) {
    const uint32_t n = (uint32_t)(p.nodes.size() / 2), ncmp = (uint32_t)(p.cmps.size() / 2);
    const std::vector<MappedNode> map = jit_map_mode(p, jit_eff_mode(cfg));
    uint32_t lut_total = 0;
    for (const MappedNode &x : map) lut_total += !x.absorbed;
    std::vector<uint8_t> pol(p.k + 1 + n, 0);  // stored polarity per ref (IMAD cells may hold ~f)
    for (uint32_t t = 0; t < n; ++t) pol[p.k + 1 + t] = map[t].pol;
    std::string s;
    s.reserve(64 * (size_t)n + 160 * (size_t)ncmp + 4096);
    char buf[320];
    snprintf(buf, sizeof buf,
             "{\n.reg .b32 %%cz;\n.reg .b32 %%cd;\n.reg .pred %%cp;\n.reg .pred %%cq;\n.reg .b32 %%cn<%u>;\nmov.b32 %%cz, 0;\n",
             std::max<uint32_t>(n, 1));
    s += buf;
    for (const std::string &m : masks) s += "mov.b32 " + m + ", 0;\n";
    auto reg = [&](uint32_t ref) -> std::string {
        if (ref == 0) return "%cz";
        if (ref <= p.k) return in_regs[ref - 1];
        return "%cn" + std::to_string(ref - p.k - 1);
    };
    std::vector<std::vector<uint32_t>> after(n + 1);
    for (uint32_t c = 0; c < ncmp; ++c) {
        const uint32_t m = std::max(p.cmps[2 * c] >> 1, p.cmps[2 * c + 1] >> 1);
        after[m > p.k ? m - p.k : 0].push_back(c);
    }
    auto emit_cmp = [&](uint32_t c) {
        const uint32_t a = p.cmps[2 * c], b = p.cmps[2 * c + 1];
        const bool inv = (((a ^ b) & 1u) != 0) != (pol[a >> 1] != pol[b >> 1]);
        const unsigned lut = inv ? 0xC3u : 0x3Cu;  // ~(a ^ b) : a ^ b on (0xF0, 0xCC)
        snprintf(buf, sizeof buf,
                 "lop3.b32 %%cd, %s, %s, %%cz, 0x%02X;\nsetp.ne.b32 %%cp, %%cd, 0;\nvote.sync.any.pred %%cq, %%cp, 0xffffffff;\n"
                 "@%%cq st.u32 [%s+%u], %%cd;\n@%%cq or.b32 %s, %s, %u;\n",
                 reg(a >> 1).c_str(), reg(b >> 1).c_str(), lut, dbuf.c_str(), 4 * c, masks[c / 32].c_str(),
                 masks[c / 32].c_str(), 1u << (c % 32));
        s += buf;
    };
    for (uint32_t c : after[0]) emit_cmp(c);
    uint32_t emitted = 0;
    for (uint32_t t = 0; t < n; ++t) {
        const MappedNode &x = map[t];
        if (x.imad) {  // FMA-pipe cell: y * m + {m, y, -1} (imad_cell)
            const std::string y = reg(x.leaf[0]), m = reg(x.leaf[1]);
            snprintf(buf, sizeof buf, "mad.lo.u32 %%cn%u, %s, %s, %s;\n", t, y.c_str(), m.c_str(),
                     x.imad_c == 0 ? m.c_str() : x.imad_c == 1 ? y.c_str() : "-1");
            s += buf;
            ++emitted;
        } else if (!x.absorbed) {
            snprintf(buf, sizeof buf, "lop3.b32 %%cn%u, %s, %s, %s, 0x%02X;\n", t,
                     x.nleaves > 0 ? reg(x.leaf[0]).c_str() : "%cz", x.nleaves > 1 ? reg(x.leaf[1]).c_str() : "%cz",
                     x.nleaves > 2 ? reg(x.leaf[2]).c_str() : "%cz", x.tt);
            s += buf;
            ++emitted;
        }
        for (uint32_t c : after[t + 1]) emit_cmp(c);
        // (never in free-warp kernels: their warps are not in step)
        if (!cfg.free_warps && !x.absorbed && lut_total > 2048 && cfg.sync_every > 0 &&
            emitted % (uint32_t)cfg.sync_every == 0)
            s += "bar.sync 0;\n";
    }
    s += "}\n";
    return s;
}

namespace {
// ---- nvJitLink (PTX -> cubin, thread-safe per handle), loaded on demand -------------------------
struct JitLink {
    void *h = nullptr;
    int (*create)(void **, uint32_t, const char **) = nullptr;
    int (*add)(void *, int, const void *, size_t, const char *) = nullptr;
    int (*complete)(void *) = nullptr;
    int (*cubin_size)(void *, size_t *) = nullptr;
    int (*cubin)(void *, void *) = nullptr;
    int (*log_size)(void *, size_t *) = nullptr;
    int (*log)(void *, char *) = nullptr;
    int (*destroy)(void **) = nullptr;
    bool tried = false, ok = false;
    bool load() {
        if (tried) return ok;
        tried = true;
        const char *cands[] = {"/usr/local/cuda/lib64/libnvJitLink.so.12", "libnvJitLink.so.12"};
        for (const char *c : cands) {
            h = dlopen(c, RTLD_NOW | RTLD_LOCAL);
            if (!h) continue;
            create = (decltype(create))dlsym(h, "__nvJitLinkCreate_12_9");
            add = (decltype(add))dlsym(h, "__nvJitLinkAddData_12_9");
            complete = (decltype(complete))dlsym(h, "__nvJitLinkComplete_12_9");
            cubin_size = (decltype(cubin_size))dlsym(h, "__nvJitLinkGetLinkedCubinSize_12_9");
            cubin = (decltype(cubin))dlsym(h, "__nvJitLinkGetLinkedCubin_12_9");
            log_size = (decltype(log_size))dlsym(h, "__nvJitLinkGetErrorLogSize_12_9");
            log = (decltype(log))dlsym(h, "__nvJitLinkGetErrorLog_12_9");
            destroy = (decltype(destroy))dlsym(h, "__nvJitLinkDestroy_12_9");
            ok = create && add && complete && cubin_size && cubin && log_size && log && destroy;
            if (ok) break;
        }
        return ok;
    }
};
JitLink g_link;
}  // namespace

// Splice-mode compile: NVRTC turns the small skeleton into PTX, the generated body replaces the
// marker line, nvJitLink assembles the result for sm_100a.
const char *jit_compile_splice(const std::vector<const JitProgram *> &ps, const JitConfig &cfg, const std::string &src,
                               std::vector<char> &cubin, std::string &log) {
    {
        std::lock_guard<std::mutex> g(g_mu);
        if (!g_nvrtc.load()) return g_nvrtc.why.c_str();
        if (!g_link.load()) return "nvJitLink (12.9) not available";
    }
    nvrtcProgram_t prog = nullptr;
    if (g_nvrtc.create(&prog, src.c_str(), "cecjit.cu", 0, nullptr, nullptr) != 0) return "nvrtcCreateProgram failed";
    const char *opts[] = {"--gpu-architecture=compute_100a", "--std=c++17", "-default-device"};
    const int rc = g_nvrtc.compile(prog, 3, opts);
    size_t ls = 0;
    g_nvrtc.log_size(prog, &ls);
    log.assign(ls, '\0');
    if (ls) g_nvrtc.log(prog, &log[0]);
    if (rc != 0) {
        g_nvrtc.destroy(&prog);
        return "NVRTC compilation failed (skeleton)";
    }
    size_t ptx_bytes = 0;
    g_nvrtc.ptx_size(prog, &ptx_bytes);
    std::string ptx(ptx_bytes, '\0');
    g_nvrtc.ptx(prog, &ptx[0]);
    g_nvrtc.destroy(&prog);
    for (size_t i = 0; i < ps.size(); ++i) {
        const JitProgram &p = *ps[i];
        const std::string marker = "//@@BODY" + std::to_string(i) + "@@";
        const size_t m = ptx.find(marker);
        if (m == std::string::npos) return "splice marker not found in PTX";
        const size_t eol = ptx.find('\n', m);
        std::vector<std::string> regs;
        {
            size_t q = m + marker.size();
            while (q < eol) {
                while (q < eol && ptx[q] == ' ') ++q;
                size_t j = q;
                while (j < eol && ptx[j] != ' ' && ptx[j] != '\r') ++j;
                if (j > q) regs.emplace_back(ptx.substr(q, j - q));
                q = j + 1;
            }
        }
        const uint32_t ncmp = (uint32_t)(p.cmps.size() / 2), M = (ncmp + 31) / 32;
        if (regs.size() != M + p.k + (ncmp ? 1 : 0)) return "splice: operand count mismatch";
        std::vector<std::string> masks(regs.begin(), regs.begin() + M), ins(regs.begin() + M, regs.begin() + M + p.k);
        const std::string dbuf = ncmp ? regs.back() : std::string("%cz");
        ptx.replace(m, eol - m, jit_body_ptx(p, cfg, masks, ins, dbuf));
    }
    while (!ptx.empty() && ptx.back() == '\0') ptx.pop_back();
    if (const char *dir = getenv("CEC_JIT_DUMP")) {
        char path[512];
        snprintf(path, sizeof path, "%s/cecjit_%016zx.ptx", dir, std::hash<std::string>()(ptx));
        if (FILE *f = fopen(path, "w")) {
            fwrite(ptx.data(), 1, ptx.size(), f);
            fclose(f);
        }
    }
    void *h = nullptr;
    const char *lopts[] = {"-arch=sm_100a"};
    if (g_link.create(&h, 1, lopts) != 0) return "nvJitLinkCreate failed";
    int r = g_link.add(h, 2 /* NVJITLINK_INPUT_PTX */, ptx.data(), ptx.size(), "cecjit.ptx");
    if (r == 0) r = g_link.complete(h);
    if (r != 0) {
        size_t es = 0;
        g_link.log_size(h, &es);
        std::string el(es, '\0');
        if (es) g_link.log(h, &el[0]);
        log += el;
        g_link.destroy(&h);
        return "nvJitLink failed";
    }
    size_t cs = 0;
    g_link.cubin_size(h, &cs);
    cubin.resize(cs);
    g_link.cubin(h, cubin.data());
    g_link.destroy(&h);
    return nullptr;
}

const char *jit_compile_cubin(const std::string &src, std::vector<char> &cubin, std::string &log) {
    {
        std::lock_guard<std::mutex> g(g_mu);
        if (!g_nvrtc.load()) return g_nvrtc.why.c_str();
    }
    nvrtcProgram_t prog = nullptr;
    if (g_nvrtc.create(&prog, src.c_str(), "cecjit.cu", 0, nullptr, nullptr) != 0) return "nvrtcCreateProgram failed";
    const char *opts[] = {"--gpu-architecture=sm_100a", "--std=c++17", "-default-device", "-lineinfo"};
    const int rc = g_nvrtc.compile(prog, 4, opts);
    size_t ls = 0;
    g_nvrtc.log_size(prog, &ls);
    log.assign(ls, '\0');
    if (ls) g_nvrtc.log(prog, &log[0]);
    if (rc != 0) {
        g_nvrtc.destroy(&prog);
        return "NVRTC compilation failed";
    }
    size_t cs = 0;
    g_nvrtc.cubin_size(prog, &cs);
    cubin.resize(cs);
    g_nvrtc.cubin(prog, cubin.data());
    g_nvrtc.destroy(&prog);
    return nullptr;
}

namespace {
std::map<std::string, std::unique_ptr<JitKernel>> g_cache;  // process-wide, keyed by structure
}

const char *jit_get_unit(const std::vector<const JitProgram *> &ps, const JitConfig &cfg, bool load, JitKernel **out) {
    if (ps.empty()) return "empty JIT unit";
    const bool bundle = ps.size() > 1;
    if (bundle && !(cfg.splice && (cfg.sync_every > 0 || cfg.free_warps)))
        return "JIT bundles need the splice mode (block-synchronous or free warps)";
    char ck[64];
    snprintf(ck, sizeof ck, "|%d,%d,%d,%d,%d,%d,%d", cfg.threads, cfg.min_blocks, cfg.sync_every, (int)cfg.fuse,
             (int)cfg.splice, (int)cfg.free_warps, cfg.ilp);
    std::string key;
    for (const JitProgram *p : ps) (key += p->key.empty() ? jit_key(*p) : p->key) += "#";
    key += ck;
    {
        std::lock_guard<std::mutex> g(g_mu);
        auto it = g_cache.find(key);
        if (it != g_cache.end() && (!load || it->second->kern)) {
            *out = it->second.get();
            return nullptr;
        }
    }
    auto t0 = std::chrono::steady_clock::now();
    if (getenv("CEC_JIT_VERIFY"))  // host emulation of every mapped body against the AIG
        for (const JitProgram *p : ps)
            if (const char *e = jit_verify_map(*p, jit_eff_mode(cfg), 64, p->nodes.size())) return e;
    const std::string src = bundle ? jit_source_bundle(ps, cfg) : jit_source(*ps[0], cfg);
    std::vector<char> cubin;
    std::string log;
    // ILP 2 (single free-warp structure): the same program is spliced into BODY0 and BODY1
    const bool ilp2 = !bundle && cfg.free_warps && cfg.splice && cfg.ilp == 2;
    const std::vector<const JitProgram *> sps = ilp2 ? std::vector<const JitProgram *>{ps[0], ps[0]} : ps;
    const char *e = (cfg.splice && (cfg.sync_every > 0 || cfg.free_warps)) ? jit_compile_splice(sps, cfg, src, cubin, log)
                                                                          : jit_compile_cubin(src, cubin, log);
    if (e) {
        static thread_local std::string msg;
        msg = std::string(e) + ": " + log.substr(0, 400);
        return msg.c_str();
    }
    if (const char *dir = getenv("CEC_JIT_DUMP")) {  // inspection: cuobjdump -sass <dir>/cecjit_*.cubin
        const size_t h = std::hash<std::string>()(key);
        char path[512];
        snprintf(path, sizeof path, "%s/cecjit_%016zx.cu", dir, h);
        if (FILE *f = fopen(path, "w")) {
            fwrite(src.data(), 1, src.size(), f);
            fclose(f);
        }
        snprintf(path, sizeof path, "%s/cecjit_%016zx.cubin", dir, h);
        if (FILE *f = fopen(path, "wb")) {
            fwrite(cubin.data(), 1, cubin.size(), f);
            fclose(f);
        }
    }
    std::unique_ptr<JitKernel> K(new JitKernel());
    K->block = cfg.threads;
    for (const JitProgram *p : ps) {
        uint32_t im = 0;
        K->lop3s.push_back(jit_lop3_count(*p, jit_eff_mode(cfg), &im));
        K->imads.push_back(im);
    }
    K->lop3 = K->lop3s[0];
    K->slices_per_pass = cfg.sync_every > 0 && !cfg.free_warps ? cfg.threads / 32 : 1;
    K->free_warps = cfg.free_warps && cfg.splice;
    K->src_bytes = src.size();
    K->cubin_bytes = cubin.size();
    if (load) {
        cudaError_t ce = cudaLibraryLoadData(&K->lib, cubin.data(), nullptr, nullptr, 0, nullptr, nullptr, 0);
        if (ce != cudaSuccess) return cudaGetErrorString(ce);
        ce = cudaLibraryGetKernel(&K->kern, K->lib, "cecjit");
        if (ce != cudaSuccess) return cudaGetErrorString(ce);
        int per_sm = 0;
        ce = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, (const void *)K->kern, K->block, 0);
        if (ce != cudaSuccess) return cudaGetErrorString(ce);
        K->blocks_per_sm = per_sm > 0 ? per_sm : 1;
    }
    K->compile_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    std::lock_guard<std::mutex> g(g_mu);
    auto &slot = g_cache[key];
    slot = std::move(K);
    *out = slot.get();
    return nullptr;
}

const char *jit_get_kernel(const JitProgram &p, const JitConfig &cfg, bool load, JitKernel **out) {
    return jit_get_unit({&p}, cfg, load, out);
}

double jit_compile_ms(const JitKernel *k) { return k ? k->compile_ms : 0.0; }
int jit_slices_per_pass(const JitKernel *k) { return k ? k->slices_per_pass : 1; }
uint32_t jit_kernel_lop3(const JitKernel *k) { return k ? k->lop3 : 0; }
bool jit_kernel_loaded(const JitKernel *k) { return k && k->kern; }
uint32_t jit_kernel_lop3_sid(const JitKernel *k, uint32_t sid) {
    return k && sid < k->lop3s.size() ? k->lop3s[sid] : 0;
}
bool jit_kernel_free(const JitKernel *k) { return k && k->free_warps; }
int jit_kernel_blocks(const JitKernel *k, int num_sms, int fallback_per_sm) {  // resident grid of a kernel
    const int per_sm = k && k->blocks_per_sm > 0 ? k->blocks_per_sm : fallback_per_sm;
    return std::max(1, num_sms) * std::max(1, per_sm);
}
int jit_kernel_block(const JitKernel *k) { return k ? k->block : 32; }
uint32_t jit_kernel_imad_sid(const JitKernel *k, uint32_t sid) {
    return k && sid < k->imads.size() ? k->imads[sid] : 0;
}

const char *jit_launch(JitKernel *K, const JItem *items, uint32_t nitems, uint32_t *ctr, unsigned long long *first,
                       unsigned long long *bound, uint32_t *neq_cnt, void *stream, int num_sms, uint32_t free_blocks) {
    if (!K || !K->kern) return "JIT kernel not loaded";
    if (nitems == 0) return nullptr;
    uint64_t grid = (uint64_t)num_sms * K->blocks_per_sm;
    const uint64_t need = K->slices_per_pass > 1 ? nitems : (nitems + (K->block / 32) - 1) / (K->block / 32);
    if (grid > need) grid = need;
    if (K->free_warps) {  // the plan partitioned the slices over exactly this many blocks (ctr = offsets)
        if (!free_blocks) return "free-warp kernel launched without its partition";
        grid = free_blocks;
    }
    void *args[] = {(void *)&items, (void *)&nitems, (void *)&ctr, (void *)&first, (void *)&bound, (void *)&neq_cnt};
    cudaError_t e = cudaLaunchKernel((const void *)K->kern, dim3((unsigned)grid), dim3(K->block), args, 0,
                                     (cudaStream_t)stream);
    return e == cudaSuccess ? nullptr : cudaGetErrorString(e);
}

}  // namespace cec
