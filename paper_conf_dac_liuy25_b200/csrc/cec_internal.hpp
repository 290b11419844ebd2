// cec_internal.hpp — structures shared by the host driver (cec_host.cpp) and the sm_100a kernels
// (sim_interp.cu). Not part of the ABI; include/cec.h is the boundary.
#pragma once
#include <cstdint>
#include <string>
#include <mutex>
#include <utility>
#include <vector>

namespace cec {

// ---- Interpreter program encoding (one uint4 = 16 B per op) ------------------------------------
// Node words live in shared-memory slots; a slot holds IV u32 words per lane of a warp
// (SLOT_BYTES = 32 * IV * 4). Offsets below are byte offsets of a slot inside the warp's region.
// AND op  (TT(n)[w] = (TT(f0)[w] ^ m0) & (TT(f1)[w] ^ m1), Alg. 1 l.10-11):
//   x = off(f0) | c0 ;  y = off(f1) | c1 ;  z = off(out) ;  w = 0
// CMP op  (XOR-compare of a pair's root words, Alg. 1 l.12-14):
//   x = off(a) | ca ;  y = off(b) | cb ;  z = OP_CMP | cmp_index ;  w = 0
constexpr uint32_t IV = 2;                       // u32 words per lane per slot
constexpr uint32_t SLOT_BYTES = 32u * IV * 4u;   // 256
constexpr uint32_t OP_CMP = 0x80000000u;
constexpr uint32_t MAX_SLOTS = 0x7FFFFFFFu / SLOT_BYTES;

struct DevWin {            // one simulation window (§III-B1) after merging
    uint32_t prog_off;     // first op in the program array
    uint32_t prog_len;     // number of ops (ANDs + CMPs)
    uint32_t k;            // number of inputs; input j lives in slot j at the start of a pass
    uint32_t const_slot;   // slot holding constant 0, or 0xFFFFFFFF if unused
    uint32_t cmp_off;      // this window's compare indices are [cmp_off, cmp_off + ncmp)
    uint32_t ncmp;
    uint32_t tt_words_lo;  // truth-table length in u32 words = max(1, 2^(k-5))
    uint32_t tt_words_hi;
};
// A slice = the words one warp carries through the window in one pass: 32 * IV words for the
// interpreter, 32 words for JIT kernels.

struct Item {              // a contiguous range of slices of one window
    uint32_t win;
    uint32_t s_begin;
    uint32_t s_end;
    uint32_t pad;
};

// ---- JIT engine (jit.cpp) -----------------------------------------------------------------------
// A window as a straight-line SSA program. Operand refs: 0 = constant 0, 1..k = input j-1,
// k+1+t = node t. nodes[2t], nodes[2t+1] = (ref << 1 | complement) of node t's fanins;
// cmps[2c], cmps[2c+1] = the two roots of the window's c-th compare.
struct JitProgram {
    uint32_t k = 0;
    std::vector<uint32_t> nodes;
    std::vector<uint32_t> cmps;
    std::string key;  // jit_key(*this) when the planner already built it (cache lookups reuse it)
};
struct JItem {             // a slice range of one JIT window instance
    uint32_t win;          // window index (bound / neq_cnt)
    uint32_t s_begin, s_end;
    uint32_t cmp_off;      // first[] index of the window's compare 0
};
struct JitKernel;
struct JitConfig {
    int threads = 512;      // threads per block
    int min_blocks = 1;     // __launch_bounds__ min blocks per SM (registers <= 64K / (threads*min_blocks))
    int sync_every = 8192;  // block-synchronous: a bar.sync every this many cells inside a body (besides the
                            // per-pass barrier); 0 = warp-independent. 512 before round 2: with IMAD cells
                            // the mid-body barriers cost more than they save (C5 32.79 -> 32.41 ms)
    int fuse = 3;           // 3-input LUT mapping: 0 none, 1 greedy (absorb single-fanout ANDs into the
                            // reader's LOP3), 2 area-flow mapping over 3-feasible cuts, 3 = 2 plus
                            // IMAD cells on the FMA pipe (jit.cpp, "Dual-pipe cells")
    bool splice = true;     // body as generated PTX spliced into an NVRTC skeleton (skips NVVM on it)
    bool free_warps = false;  // single small structure: static per-warp slice partition, no barriers
    int ilp = 1;              // free warps: slices evaluated per pass (2 = two interleaved body copies)
};
struct LaunchGroup {       // windows sharing one kernel launch
    uint32_t nslots;       // interpreter: slots per warp in this launch
    uint32_t item_off, nitems;
    JitKernel *jit = nullptr;  // non-null: a JIT structure group (items index DevPlan::jitems)
    uint64_t lop3_words = 0;   // executed LOP3 x u32 words of the group (CEC_PROFILE_GROUPS report)
    uint32_t nwin = 0, max_k = 0, nodes = 0;
    uint32_t free_blocks = 0;  // free-warp JIT kernel: grid size the slices were partitioned over
    uint32_t joff_off = 0;     // ... and its per-warp item offsets (DevPlan::joff, free_blocks*warps+1)
};

// Device buffers of one plan.
struct DevPlan {
    DevWin *wins = nullptr;
    uint4 *prog = nullptr;
    Item *items = nullptr;
    unsigned long long *first = nullptr;  // [ncmp] minimum mismatching merged pattern index
    unsigned long long *bound = nullptr;  // [nwin] early-exit bound (all pairs NEQ below it)
    uint32_t *neq_cnt = nullptr;          // [nwin]
    uint32_t *item_ctr = nullptr;         // [ngroups]
    JItem *jitems = nullptr;
    uint32_t *joff = nullptr;             // free-warp groups: per-warp CSR offsets into jitems
};

// Per-context cache of device blocks and one pinned host staging buffer (sim_interp.cu): a plan takes
// one device block for all its buffers and returns it on free, so repeated calls do no
// cudaMalloc/cudaFree (cudaFree synchronises the device). Shared (refcounted) by the context and
// its live plans, so a plan may outlive the context.
struct DevPool {
    std::mutex mu;
    std::vector<std::pair<void *, size_t>> free_blocks;
    void *pinned = nullptr;
    size_t pinned_bytes = 0;
    void *pinned_ev = nullptr;  // last H2D out of the staging buffer
    const char *get(size_t bytes, void **p, size_t *cap);
    void put(void *p, size_t cap);
    const char *staging(size_t bytes, void **host);  // waits for the previous H2D out of it
    const char *staged(void *stream);                // records the H2D just issued
    ~DevPool();
};

// supp_gpu.cu: a2 supports of all pairs (sorted PI lists saturating at cap = k_max + 1). The per-node
// table (AIG-only) is computed into *table on first use and reused while table->cap == cap.
struct NodeSupports {
    uint32_t *lists = nullptr, *cnt = nullptr;  // one cudaMalloc block, N x cap + N
    uint32_t cap = 0, launches = 0;
};
const char *gpu_supports(DevPool &pool, const uint32_t *d_f0, const uint32_t *d_f1, const uint32_t *d_level_ids,
                         const std::vector<uint32_t> &level_off, uint32_t I, uint32_t N, uint32_t cap,
                         const std::vector<uint2> &roots, std::vector<uint32_t> &lists_out,
                         std::vector<uint32_t> &cnt_out, void *stream, uint32_t *launches, NodeSupports *table);
// supp_gpu.cu: AND-cone sizes |TFI(a) u TFI(b)| of pairs (the cost-aware merge's estimates);
// UINT32_MAX where the cone does not fit the block's shared-memory walk (the host walks those).
const char *gpu_cones(DevPool &pool, const uint32_t *d_f0, const uint32_t *d_f1, uint32_t I,
                      const std::vector<uint2> &roots, std::vector<uint32_t> &cone_out, void *stream);

// jit.cpp
std::string jit_key(const JitProgram &p);
std::string jit_source(const JitProgram &p, const JitConfig &cfg);
const char *jit_compile_cubin(const std::string &src, std::vector<char> &cubin, std::string &log);
const char *jit_get_kernel(const JitProgram &p, const JitConfig &cfg, bool load, JitKernel **out);
// several structures in one kernel (items carry window | sid << 20), see jit_source_bundle
const char *jit_get_unit(const std::vector<const JitProgram *> &ps, const JitConfig &cfg, bool load, JitKernel **out);
uint32_t jit_kernel_lop3_sid(const JitKernel *k, uint32_t sid);
bool jit_kernel_loaded(const JitKernel *k);  // true once the cubin is loaded (kernel handle set)
double jit_compile_ms(const JitKernel *k);
int jit_slices_per_pass(const JitKernel *k);
uint32_t jit_kernel_lop3(const JitKernel *k);
uint32_t jit_lop3_count(const JitProgram &p, int mode, uint32_t *imads = nullptr);
uint32_t jit_kernel_imad_sid(const JitKernel *k, uint32_t sid);
int jit_eff_mode(const JitConfig &cfg);
const char *jit_launch(JitKernel *K, const JItem *items, uint32_t nitems, uint32_t *ctr, unsigned long long *first,
                       unsigned long long *bound, uint32_t *neq_cnt, void *stream, int num_sms, uint32_t free_blocks = 0);
bool jit_kernel_free(const JitKernel *k);
int jit_kernel_blocks(const JitKernel *k, int num_sms, int fallback_per_sm);
int jit_kernel_block(const JitKernel *k);

// cuts_gpu.cu
uint32_t gpu_cuts_max_C();
const char *gpu_common_cuts(const uint32_t *d_f0, const uint32_t *d_f1, uint32_t N,
                            const std::vector<uint32_t> &fanout, const std::vector<uint32_t> &level,
                            const std::vector<uint32_t> &repr_of, const std::vector<uint32_t> &pis_needed,
                            const std::vector<std::vector<uint32_t>> &el_lists, const std::vector<uint32_t> &repr,
                            const std::vector<uint32_t> &member, uint32_t k_l, uint32_t C, int pass, uint32_t max_cuts,
                            void *stream, int num_sms, std::vector<uint32_t> &cut_counts,
                            std::vector<uint32_t> &cut_leaves_flat);

// sim_simt.cu — the paper's Alg. 1 (simulation table in HBM, rounds x levels) for comparison
struct SimtPlan {
    uint32_t E = 0;                 // words per row per round (0 = plan does not use this engine)
    uint64_t rounds = 0, rows = 0;
    uint4 *d_simt = nullptr;        // rows x E words
    bool simt_in_workspace = false; // d_simt is the caller's workspace (cec_opts.workspace): not freed
    uint4 *d_inputs = nullptr;      // {row, window, j, 0}
    uint4 *d_nodes = nullptr;       // by level: {row, row_f0 | c0 << 31, row_f1 | c1 << 31, window}
    uint4 *d_pairs = nullptr;       // {row_a | ca << 31, row_b | cb << 31, window, cmp}
    unsigned long long *d_ttw = nullptr;  // words of each window's truth table
    uint32_t n_inputs = 0, n_pairs = 0;
    std::vector<uint32_t> level_off;
    std::vector<uint4> h_inputs, h_nodes, h_pairs;
    std::vector<unsigned long long> h_ttw;
};
const char *launch_simt(const SimtPlan &S, unsigned long long *first, uint32_t ncmp, void *stream, int num_sms,
                        uint32_t *launches);

// reduce_gpu.cu: miter reduction (merge + strash rebuild) over a host topological batch schedule
const char *gpu_reduce(const uint32_t *d_f0, const uint32_t *d_f1, uint32_t I, uint32_t N, const std::vector<uint32_t> &sub,
                       const std::vector<uint32_t> &batch_ids, const std::vector<uint32_t> &batch_off, void *stream,
                       int num_sms, DevPool *pool, std::vector<uint32_t> &new_fanins, std::vector<uint32_t> &image,
                       uint32_t *launches, float *kernel_ms);

// classes_gpu.cu: partial simulation -> exact equivalence classes -> (repr, member, phase) pairs
const char *gpu_classes(const uint32_t *d_f0, const uint32_t *d_f1, const uint32_t *d_level_ids,
                        const std::vector<uint32_t> &level_off, uint32_t I, uint32_t N, uint32_t Wr, uint64_t seed,
                        uint32_t Wc, const uint32_t *h_words, uint32_t cap, void *stream, int num_sms,
                        DevPool *pool, uint32_t *total_out, std::vector<uint32_t> &repr,
                        std::vector<uint32_t> &member, std::vector<uint8_t> &phase, uint32_t *launches,
                        float *kernel_ms);

// sim_random.cu
const char *random_sim(const uint32_t *d_f0, const uint32_t *d_f1, const uint32_t *d_level_ids,
                       const std::vector<uint32_t> &level_off, uint32_t I, uint32_t N, uint32_t W, uint64_t seed,
                       uint32_t *d_tt, unsigned long long *d_sig, uint8_t *d_phase, void *stream, int num_sms,
                       uint32_t *launches, bool pi_words_given);

// sim_interp.cu
// Side streams: independent launch groups (different window structures) run concurrently, so the
// tail of one persistent grid overlaps the next and small groups do not serialise.
constexpr int NAUX_MAX = 32;
struct AuxStreams {
    int n = 0;                 // side streams in use (CEC_SIDE_STREAMS, default 4)
    void *s[NAUX_MAX] = {};
    void *fork = nullptr;
    void *join[NAUX_MAX] = {};
    bool ok = false;
};
const char *aux_create(AuxStreams &a);
void aux_destroy(AuxStreams &a);

// peer.cu — a10 over NVLink peer memory: rank 0's exchange block is the
// home of first[] / bound[] / neq_cnt[]; every rank's kernels update it directly.
constexpr int PEER_MAX = 8;
constexpr int PEER_EPOCH = PEER_MAX;      // own-block word: this rank's barrier epoch
constexpr int PEER_ERR = PEER_MAX + 1;    // own-block word: 1 = a barrier timed out
constexpr size_t PEER_HDR_BYTES = 256;    // slots + epoch + error flag, padded
struct PeerPtrs {
    uint32_t *slots[PEER_MAX];            // peer r's block (its arrival slots first), mapped here
};
struct PeerState {                        // per context
    bool on = false;
    int rank = 0, world = 1;
    uint32_t cap_cmp = 1u << 20, cap_win = 1u << 18;  // per-run capacity of the home arrays
    void *own = nullptr;                  // this rank's block (cudaMalloc, IPC-exported)
    size_t bytes = 0;
    void *peer[PEER_MAX] = {};            // every rank's block as mapped in this process
    void *opened[PEER_MAX] = {};          // IPC mappings to close
    uint32_t gen = 0;                     // bumped per import (invalidates captured graphs)
    uint64_t timeout_ns = 60000000000ull; // barrier wait before the error flag (CEC_PEER_TIMEOUT_S)
    void (*host_barrier)(void *) = nullptr;  // emulation of several ranks on ONE device (tests):
    void *host_user = nullptr;               // barriers become stream sync + this host callback
};
struct PeerRun {                          // what one run needs (passed into launch_run)
    bool on = false;
    int rank = 0, world = 1;
    PeerPtrs slots{};
    uint32_t *own = nullptr;
    unsigned long long *home_first = nullptr, *home_bound = nullptr;
    uint32_t *home_neq = nullptr;
    unsigned long long *local_first = nullptr;  // the plan's first[]: receives the gathered result
    uint64_t timeout_ns = 60000000000ull;
    void (*host_barrier)(void *) = nullptr;
    void *host_user = nullptr;
};
size_t peer_block_bytes(uint32_t cap_cmp, uint32_t cap_win);
const char *peer_export(PeerState &ps, int device, int rank, int world, void *blob128);
const char *peer_import(PeerState &ps, int device, int rank, int world, const void *blobs);
void peer_close(PeerState &ps);
PeerRun peer_run_of(const PeerState &ps, unsigned long long *local_first);
const char *peer_barrier_launch(const PeerRun &pr, void *stream);
const char *peer_gather_launch(const PeerRun &pr, uint32_t n, void *stream);
const char *peer_error(const PeerState &ps, void *stream, bool *timed_out);

// One run of a plan: reset, every launch group (side streams forked/joined). With pr->on the window
// kernels take rank 0's home arrays (d's first/bound/neq_cnt are replaced), wrapped in the peer
// barriers and followed by the gather into d.first. no_join: the caller's stream does NOT wait for
// the side streams at the end (the pipelined call's earlier chunks: the next chunk's kernels touch
// only their own arrays, so they may start while this chunk's side-stream kernels finish; the last
// chunk joins, and side streams run in order, so its join covers every chunk).
// sweep_ev (optional, two events): recorded on the caller's stream right before the first window
// kernel (after the reset) and right after the side streams joined, i.e. around the window kernels
// only (not the reset, peer barriers, gather or all-reduce); inside a graph capture as external
// event-record nodes, so every replay re-records them.
const char *launch_run(const DevPlan &d, const std::vector<LaunchGroup> &groups, uint32_t nwin, uint32_t ncmp,
                       void *stream, int num_sms, uint32_t *launches, AuxStreams *aux, const PeerRun *pr = nullptr,
                       bool no_join = false, void *const *sweep_ev = nullptr);
const char *graph_capture_run(const DevPlan &d, const std::vector<LaunchGroup> &groups, uint32_t nwin, uint32_t ncmp,
                              void *stream, int num_sms, uint32_t *launches, AuxStreams *aux, void **exec_out,
                              const PeerRun *pr = nullptr, void *const *sweep_ev = nullptr);
const char *graph_launch(void *exec, void *stream);
void graph_destroy(void *exec);
const char *dev_alloc(void **p, size_t bytes);
const char *dev_free(void *p);
const char *h2d(void *dst, const void *src, size_t bytes, void *stream);
const char *d2h(void *dst, const void *src, size_t bytes, void *stream);
const char *dev_memset(void *dst, int v, size_t bytes, void *stream);
const char *stream_sync(void *stream);
const char *dev_init(int device, void **own_stream, int *num_sms);
const char *stream_destroy(void *stream);
const char *event_create(void **ev);
const char *event_record(void *ev, void *stream);
const char *event_elapsed(float *ms, void *a, void *b);
void event_destroy(void *ev);
uint32_t interp_max_slots_per_warp();

}  // namespace cec
