/*
 * cec.h — C ABI of the B200 exhaustive-simulation CEC hot path (libcec.so).
 *
 * The boundary follows the paper's problem statement: given a combinational And-Inverter Graph
 * holding two circuits with shared PIs (a miter, §II-B) and candidate node pairs,
 * decide for each pair equivalent / not equivalent with a counter-example (§III-A,
 * footnote 1 at :69) / undecided (§III-D); and, for pairs whose support is too large,
 * check their local functions on a common cut (§III-C1).
 *
 * Conventions used by every call
 *  - Node ids: 0 = constant 0; 1..num_pis = PIs in input order; num_pis+1 .. num_pis+num_ands =
 *    AND nodes. Every AND's fanin ids are smaller than its own id (AIGER-binary order), so the id
 *    order is a topological order.
 *  - A literal is 2*id + complement ("signals can be optionally inverted").
 *  - Pattern index / truth-table convention (§II-A): for a window with inputs
 *    S[0] < S[1] < ... < S[k-1] (increasing node id), pattern i assigns input S[j]
 *    the value of bit j of i. CEX indices are given in the PAIR'S OWN support order with every
 *    non-support PI = 0, and are the MINIMUM mismatching index (canonical CEX).
 *  - Ownership: the caller owns every array passed in and every output array; the library copies
 *    what it keeps. A context owns its device buffers and plans. A context is not thread-safe.
 *  - Errors: every call returns cec_status; no C++ exception crosses the ABI. On error,
 *    cec_last_error(ctx) returns a NUL-terminated message (valid until the next call on ctx).
 *  - No CPU fallback: simulation entry points need a CUDA device and return CEC_E_CUDA without
 *    one. A context created with opts.device = -1 is "host only": it can load, validate and plan
 *    (cec_pair_support, cec_plan_*_info) but every simulation call returns CEC_E_CUDA.
 */
#ifndef CEC_H
#define CEC_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define CEC_ABI_VERSION 2  /* 2: cec_stats.imad_words */
#define CEC_NO_CEX UINT64_MAX

typedef struct cec_ctx cec_ctx;
typedef struct cec_plan cec_plan;

typedef enum {
    CEC_OK = 0,
    CEC_E_ARG = 1,    /* bad argument (NULL pointer, literal out of range, k_max > 63, ...) */
    CEC_E_AIG = 2,    /* malformed AIG: fanin id >= own id, literal out of range */
    CEC_E_CUT = 3,    /* a local-check leaf set is not a cut of its roots */
    CEC_E_NOMEM = 4,  /* host or device allocation failed, or a window exceeds on-chip capacity */
    CEC_E_CUDA = 5,   /* CUDA error, or no CUDA device (host-only context) */
    CEC_E_NCCL = 6,   /* NCCL error in the cross-GPU reduction */
    CEC_E_NOCEX = 7,  /* cec_get_cex on a pair that was not NOT_EQUIVALENT */
    CEC_E_STATE = 8   /* call order violated (e.g. cec_get_cex before any cec_sim_exhaustive) */
} cec_status;

typedef enum {
    CEC_BAD_CUT = -1,          /* local check only: the leaves are not a cut of the pair */
    CEC_UNDECIDED = 0,         /* support above k_max (global) or local functions differ (local) */
    CEC_EQUIVALENT = 1,
    CEC_NOT_EQUIVALENT = 2     /* global check only: a counter-example exists */
} cec_verdict;

typedef enum {
    CEC_MERGE_OFF = 0,
    CEC_MERGE_PAPER = 1, /* lexicographic sort + greedy consecutive merge, union <= k_s */
    CEC_MERGE_COST = 2   /* same sort and greedy pass, but a merge is taken only if it does not
                            increase the estimated work (nodes x 2^k); results are identical (Q8) */
} cec_merge_policy;

typedef enum {
    CEC_ENGINE_AUTO = 0,
    CEC_ENGINE_INTERP = 1, /* schedule interpreter: values in shared memory slots */
    CEC_ENGINE_JIT = 2,    /* per-window-structure register-resident kernel compiled with NVRTC */
    CEC_ENGINE_SIMT = 3    /* the paper's Alg. 1: simulation table in HBM, rounds of
                              E words, one launch per topological level; global checks on one GPU
                              only (world = 1); table size M from env CEC_SIMT_MB (default 16384) */
} cec_engine;

typedef struct {
    uint32_t num_pis;
    uint32_t num_ands;
    uint32_t num_pos;
    const uint32_t *fanin_lits; /* [2*num_ands]: AND i (id num_pis+1+i) = (lit[2i], lit[2i+1]) */
    const uint32_t *po_lits;    /* [num_pos] (informational; pairs are passed explicitly) */
} cec_aig;

typedef struct {
    int32_t device;            /* CUDA device ordinal; -1 = host-only context (no simulation) */
    int32_t rank, world;       /* world > 1: SPMD over `world` GPUs; every rank passes the same
                                  AIG, pairs and options; rank r simulates its contiguous share of
                                  every window's pattern slices */
    const void *nccl_unique_id;/* 128-byte ncclUniqueId for world >= 1 (the caller bootstraps it,
                                  e.g. through torch.distributed): one ncclAllReduce(min) of the
                                  per-pair first-mismatch indices makes the results identical on
                                  every rank. NULL with world > 1 = shard-only mode: no collective;
                                  results cover this rank's slices only (NOT_EQUIVALENT iff a CEX
                                  lies in them, with the minimum such index) and the caller combines
                                  ranks by taking the per-pair minimum index */
    void *stream;              /* cudaStream_t to launch on, or NULL for the library's own stream */
    uint32_t k_max;            /* exhaustive support limit, <= 63. Default 32 (= k_P) */
    uint32_t k_s;              /* window-merge threshold; 0 = k_max */
    int32_t merge;             /* cec_merge_policy; default CEC_MERGE_PAPER */
    int32_t engine;            /* cec_engine; default CEC_ENGINE_AUTO */
    void *workspace;           /* caller-owned device memory for CEC_ENGINE_SIMT's simulation table:
                                  Alg. 1's memory budget M. E = the largest
                                  power of two with E x rows x 4 B <= workspace_bytes; the table
                                  lives in the workspace (not freed by the library; the caller keeps
                                  it alive and unused while plans of the context run). NULL = the
                                  library allocates M itself (CEC_SIMT_MB, default 16 GiB). The
                                  product engines (JIT, interpreter) keep truth tables on chip and
                                  ignore it. */
    uint64_t workspace_bytes;
    uint64_t reserved[4];      /* must be zero */
} cec_opts;

typedef struct {
    uint64_t node_patterns;    /* W: sum over simulated windows of (#AND nodes) x (#patterns
                                  simulated by this rank), after merging */
    uint64_t node_patterns_all;/* same, all ranks together */
    uint32_t num_windows;      /* windows after merging */
    uint32_t max_k;            /* largest window input count */
    uint32_t max_slots;        /* largest on-chip live set (interpreter slots) */
    uint32_t num_launches;     /* kernel launches of the last run */
    float kernel_ms;           /* device time of the last run (first launch .. reduction done) */
    float host_prep_ms;        /* host planning time of the last plan */
    uint64_t h2d_bytes;        /* bytes copied host->device by the last plan (schedules, items) */
    uint64_t d2h_bytes;        /* bytes copied device->host by the last results read-back */
    float jit_ms;              /* NVRTC compile + load time spent by the last plan (0 if cached) */
    uint32_t jit_kernels;      /* distinct window structures compiled for the last plan */
    uint32_t jit_windows;      /* windows of the last plan run by JIT kernels (rest: interpreter) */
    uint64_t lop3_words;       /* LOP3 instructions x u32 words this rank executes per run for the AND
                                  nodes: mapped 3-input LUTs for JIT windows (a LUT may evaluate
                                  two ANDs), one per AND for interpreter windows */
    uint64_t imad_words;       /* IMAD cells x u32 words this rank executes per run: AND nodes of JIT
                                  windows evaluated on the FMA pipe (mad.lo.u32 with a word-uniform
                                  input word, 0 or ~0; jit.cpp "Dual-pipe cells") */
} cec_stats;

/* Fill *opts with the defaults above. */
void cec_default_opts(cec_opts *opts);

/* Create a context: copy and validate the AIG (CEC_E_AIG if any fanin id >= own id or a literal
 * is out of range), select the device, and when opts->world > 1 create the NCCL communicator
 * (collective: every rank must call it). *ctx is set only on CEC_OK. */
cec_status cec_load_aig(cec_ctx **ctx, const cec_aig *aig, const cec_opts *opts);

/* Replace the context's AIG by the next version of the miter (the miter is
 * reduced after each phase and the next phase works on the reduced one), keeping everything that
 * does not depend on the AIG: device, streams, host workers, device buffer pool, compiled JIT
 * kernels, NCCL communicator / peer mappings (so a P -> G -> L* flow pays no context creation per
 * phase). Validation as in cec_load_aig; a rejected AIG (CEC_E_AIG / CEC_E_ARG) leaves the context
 * unchanged. k_max / k_s: the new limits (0 = keep; k_s = 0 with k_max > 0 means k_s = k_max).
 * Blocking (waits for the context's stream). Drops what the old AIG produced: the device copy of
 * the AIG, the per-node support table, the last global check (cec_get_cex -> CEC_E_STATE).
 * Collective when world > 1 in the sense that every rank must reload the same AIG. */
cec_status cec_reload_aig(cec_ctx *ctx, const cec_aig *aig, uint32_t k_max, uint32_t k_s);

/* Global exhaustive check of num_pairs literal pairs (Alg. 1 :89-108).
 * For a pair with k = |supp(a) U supp(b)| <= k_max the verdict is exact: EQUIVALENT, or
 * NOT_EQUIVALENT with cex_index_out = the minimum mismatching pattern in the pair's own support
 * order. k > k_max (or k > 41: more than 2^41 patterns) gives UNDECIDED and CEC_NO_CEX (the caller
 * may fall back to local cuts).
 * lit_a == lit_b -> EQUIVALENT; lit_a == lit_b ^ 1 -> NOT_EQUIVALENT at index 0.
 * verdict_out / cex_index_out / k_out are caller-owned host arrays of num_pairs (cex_index_out and
 * k_out may be NULL). Blocking: returns after the kernels, the cross-GPU reduction and the copy
 * back. Windows are merged per opts->merge. */
cec_status cec_sim_exhaustive(cec_ctx *ctx, uint32_t num_pairs, const uint32_t *lit_a, const uint32_t *lit_b,
                              int32_t *verdict_out, uint64_t *cex_index_out, uint32_t *k_out);

/* Local function checks (§III-C1). Check q compares lit_a[q] and lit_b[q] as
 * functions of the leaves cut_leaves[cut_off[q] .. cut_off[q+1]) (node ids > 0, any order, taken in
 * increasing id; at most k_max and at most 24 leaves; CEC_E_ARG otherwise). verdict_out[q] = EQUIVALENT if the two local
 * functions are identical; UNDECIDED if they differ (the difference may be an SDC, so
 * no CEX is produced); CEC_BAD_CUT if the backward traversal from a root reaches a PI that is not a
 * leaf, in which case the call returns CEC_E_CUT after filling every other verdict. */
cec_status cec_check_local_cuts(cec_ctx *ctx, uint32_t num_checks, const uint32_t *lit_a, const uint32_t *lit_b,
                                const uint32_t *cut_off, const uint32_t *cut_leaves, int32_t *verdict_out);

/* Partial random simulation (PAPER.md:41 §II-B, :61, :183): simulate every node on num_words*32
 * random patterns (PI id i, word w gets the low 32 bits of splitmix64(seed ^ (i << 32) ^ w)) on the
 * GPU and write one 64-bit signature per node id to sig_out[1+num_pis+num_ands], canonical under
 * complement: phase_out[id] = 1 if the node evaluates to 1 on pattern 0 and was complemented
 * before hashing. Nodes with equal signatures are candidate-equivalent (equivalence classes,
 * representative = minimum id); a signature is a filter, never a proof. */
cec_status cec_sim_random(cec_ctx *ctx, uint32_t num_words, uint64_t seed, uint64_t *sig_out, uint8_t *phase_out);

/* Same as cec_sim_random with caller-chosen patterns (e.g. counter-examples, "CEX
 * patterns for splitting the class of a disproved pair"): PI id i+1 takes the num_words u32 words
 * pi_words[i*num_words .. (i+1)*num_words). */
cec_status cec_sim_patterns(cec_ctx *ctx, uint32_t num_words, const uint32_t *pi_words, uint64_t *sig_out,
                            uint8_t *phase_out);

/* Equivalence classes from partial simulation, on the GPU (§II-B "nodes with identical
 * partial truth tables are put into the same equivalence class"; :61/:183; :187 counter-example
 * patterns split classes). Every node is simulated on 32*(num_words +
 * num_pattern_words) patterns: first num_words random words per PI (PI id i, word w: low 32 bits
 * of splitmix64(seed ^ (i << 32) ^ w), as in cec_sim_random), then the caller's words (PI id i+1
 * takes pi_words[i*num_pattern_words .. (i+1)*num_pattern_words), e.g. CEXs packed LSB-first).
 * Nodes whose value vectors are equal or complementary form one class (exactly: rows are compared,
 * a signature collision never merges classes); representative = minimum id (const 0 and PIs may
 * represent, only AND nodes are members). Output, ordered by member id: (repr_out[q], member_out[q],
 * phase_out[q] = 1 if the member is the representative's complement); *num_pairs_out = the total
 * number of pairs, of which the first min(total, cap) are written to the caller-owned arrays. */
cec_status cec_sim_classes(cec_ctx *ctx, uint32_t num_words, uint64_t seed, uint32_t num_pattern_words,
                           const uint32_t *pi_words, uint32_t cap, uint32_t *num_pairs_out, uint32_t *repr_out,
                           uint32_t *member_out, uint8_t *phase_out);

/* Host cut generator for local checks (Eq. 1, Table I, similarity-guided
 * selection). For candidate pairs q (repr[q] < member[q], node ids; member equivalent to repr up to
 * complement), enumerate priority cuts (<= C per node, <= k_l <= 24 leaves, dominated cuts dropped,
 * Table I order of pass_id in {0,1,2}; members ranked first by similarity to their
 * representative's cuts) over the TFI of all pairs, and return each pair's common cuts u|v
 * (<= k_l leaves, smallest first, at most max_cuts): pair q's cuts are [pair_cut_off[q],
 * pair_cut_off[q+1]) and cut t's leaves (node ids, increasing) are leaves[cut_off[t] ..
 * cut_off[t+1]). Caller-owned outputs: pair_cut_off[npairs+1], cut_off[npairs*max_cuts+1],
 * leaves[npairs*max_cuts*k_l]. Host-only (no GPU needed); feed the cuts to cec_check_local_cuts. */
cec_status cec_common_cuts(cec_ctx *ctx, uint32_t npairs, const uint32_t *repr, const uint32_t *member,
                           uint32_t k_l, uint32_t C, int32_t pass_id, uint32_t max_cuts, uint32_t *pair_cut_off,
                           uint32_t *cut_off, uint32_t *leaves);

/* One cut generation + local checking pass, Alg. 2:
 * the priority cuts of cec_common_cuts (same definition, same cuts) are enumerated level by level
 * in the enumeration levels of Eq. (2) (the nodes of a level in parallel), and as soon as a
 * member's cuts exist, the common cuts of its pair (member[q] with repr[q], relative phase
 * phase[q]: the pair is the literals 2*repr and 2*member ^ phase) enter a buffer that is flushed to
 * the local-check kernels (cec_check_local_cuts semantics) whenever it holds
 * buffer_checks checks; the GPU checks one buffer while the host enumerates the next levels.
 * verdict_out[q] = EQUIVALENT if any common cut of pair q proves it, else UNDECIDED.
 * *num_checks_out = checks issued. Optional check log (NULL allowed), in issue order, with caller
 * capacities npairs*max_cuts (+1 for check_cut_off) and npairs*max_cuts*k_l leaves:
 * check_pair[i], leaves check_leaves[check_cut_off[i] .. check_cut_off[i+1]), check_verdict[i].
 * Results do not depend on buffer_checks. CEC_E_CUDA without a device. */
cec_status cec_local_pass(cec_ctx *ctx, uint32_t npairs, const uint32_t *repr, const uint32_t *member,
                          const uint8_t *phase, uint32_t k_l, uint32_t C, int32_t pass_id, uint32_t max_cuts,
                          uint32_t buffer_checks, int32_t *verdict_out, uint32_t *num_checks_out,
                          uint32_t *check_pair, uint32_t *check_cut_off, uint32_t *check_leaves,
                          int32_t *check_verdict);

/* Miter reduction on the GPU ("reduces the miter by merging the proved equivalent
 * pairs", :185, :187). Merge q redirects every fanout of AND node member[q]
 * to the literal repr_lit[q] (a proved equivalence; repr_lit[q] >> 1 < member[q], representative =
 * lower id; each member listed once); then the AIG is rebuilt with structural hashing: every
 * AND in increasing id gets image = new(repr) if merged, else AND(new(f0), new(f1)) with
 * x&0 = 0, x&1 = x, x&x = x, x&!x = 0 and one node per normalised fanin pair (a < b), new ids in
 * creation order (AIGER-binary order again). Outputs (caller-owned host arrays):
 * *new_num_ands; new_fanin_lits[2 * new_num_ands] (capacity 2 * num_ands suffices: the result never
 * grows); image_out[1 + num_pis + num_ands] (NULL allowed) = the new literal of every old node id;
 * lits[num_lits] (in/out, NULL allowed when num_lits = 0): old literals mapped to new ones (e.g.
 * the PO pairs). PIs keep their ids. CEC_E_ARG for a bad merge list; CEC_E_CUDA without a device.
 * The context keeps the old AIG: load the result with cec_load_aig. */
cec_status cec_reduce(cec_ctx *ctx, uint32_t num_subst, const uint32_t *member, const uint32_t *repr_lit,
                      uint32_t *new_num_ands, uint32_t *new_fanin_lits, uint32_t *image_out, uint32_t num_lits,
                      uint32_t *lits);

/* Counter-example of pair `pair_idx` of the most recent cec_sim_exhaustive / cec_plan_results:
 * pi_values_out[i] = value of PI id i+1 (0/1): PI S[j] = bit j of the CEX index, every other PI 0.
 * CEC_E_NOCEX unless that pair was NOT_EQUIVALENT; CEC_E_STATE before any global check. */
cec_status cec_get_cex(cec_ctx *ctx, uint32_t pair_idx, uint8_t *pi_values_out);

/* Structural support of {var(lit_a), var(lit_b)}: writes min(k, cap) PI ids in
 * increasing order to support_out (may be NULL when cap = 0) and returns k via *k_out. */
cec_status cec_pair_support(cec_ctx *ctx, uint32_t lit_a, uint32_t lit_b, uint32_t *support_out, uint32_t cap,
                            uint32_t *k_out);

/* ---- Plans: split cec_sim_exhaustive into host planning, device run and result read-back, so a
 * caller can time the device part with the inputs already resident in HBM. ------------------------ */

/* Host planning for a global check: supports, windows, merging, schedules; uploads the schedules.
 * A host-only context plans without uploading. */
cec_status cec_plan_exhaustive(cec_ctx *ctx, uint32_t num_pairs, const uint32_t *lit_a, const uint32_t *lit_b,
                               cec_plan **plan);
/* Launch the plan's kernels (and the cross-GPU reduction) on the context stream; asynchronous. */
cec_status cec_plan_run(cec_ctx *ctx, cec_plan *plan);
/* Wait for the plan, copy the results back and decode them exactly as cec_sim_exhaustive does. */
cec_status cec_plan_results(cec_ctx *ctx, cec_plan *plan, int32_t *verdict_out, uint64_t *cex_index_out,
                            uint32_t *k_out);
/* Plan shape: windows after merging, W for one full run, largest k and live set. */
cec_status cec_plan_info(const cec_plan *plan, uint32_t *num_windows, uint64_t *node_patterns, uint32_t *max_k,
                         uint32_t *max_slots);
/* Kernel timing of a plan (the denominator of the kernels' roofline fraction in bench.py). With
 * cec_plan_sweep_timing(plan, 1), every run records two CUDA events on the context's stream, right
 * before the first window kernel and right after the side streams joined: the sweep itself,
 * without the reset kernel, peer barriers / gather or all-reduce and the graph launch latency. Off
 * by default: the two event nodes add a few microseconds to a captured run (C2: ~7 us of 38).
 * cec_plan_sweep_ms = that interval for the last completed run (the caller synchronises first).
 * CEC_E_STATE: the last run was not timed / has not completed, or a plan of the SIMT engine. */
cec_status cec_plan_sweep_timing(cec_plan *plan, int on);
cec_status cec_plan_sweep_ms(const cec_plan *plan, float *ms);
/* Per-window description, for tests of the host logic: window w's inputs (node ids, increasing),
 * its AND-node count and its pair indices. Arrays may be NULL to query sizes only. */
cec_status cec_plan_window(const cec_plan *plan, uint32_t w, uint32_t *inputs, uint32_t *k, uint32_t *num_nodes,
                           uint32_t *pairs, uint32_t *num_pairs);
void cec_plan_free(cec_plan *plan);

/* The CUDA stream the context launches on (cudaStream_t). */
void *cec_stream(cec_ctx *ctx);
/* Statistics of the last run on this context. */
cec_status cec_get_stats(cec_ctx *ctx, cec_stats *stats);

/* Create a 128-byte ncclUniqueId (rank 0 calls it and shares the bytes with the other ranks, e.g.
 * through torch.distributed) using the NCCL library libcec loads on demand. CEC_E_NCCL if NCCL is
 * unavailable. */
cec_status cec_nccl_unique_id(void *out128);

/* Cross-GPU reduction over NVLink peer memory instead of NCCL (SURVEY.md §8(e) "B200-native
 * option", §8(f) NEXT-4): the a10 min-reduction of first_idx fused into the compare path, with
 * cross-GPU bounded early exit (Q9).
 * Setup is collective over the `world` ranks of contexts loaded with the same opts.world (2..8):
 *   1. every rank calls cec_peer_export: allocates its exchange block (~11 MB of device memory:
 *      arrival slots, and home arrays for up to 2^20 compares and 2^18 windows per run) and writes a
 *      CEC_PEER_BLOB_BYTES blob (CUDA IPC handle, pid, device, rank) into blob_out;
 *   2. the caller all-gathers the blobs in rank order (e.g. torch.distributed.all_gather_object);
 *   3. every rank calls cec_peer_import with the world blobs (world x 128 bytes, rank order): peer
 *      blocks of other processes are mapped with CUDA IPC, blocks of the same process used directly.
 * From then on every cec_plan_run / cec_sim_exhaustive / cec_check_local_cuts of this context runs
 * in peer mode: rank 0's block is the home of the run's first-mismatch indices, bounds and counters;
 * every rank's window kernels update it with system-scope atomics on the (rare) mismatch path and
 * read its bounds for early exit; device-side barriers (one-warp kernels, no host round trip; CUDA
 * graph safe) order reset -> kernels -> gather -> next run. Results are identical to the NCCL path
 * (the same per-pair minimum index) and identical on every rank. Every rank must issue the same
 * sequence of runs (SPMD, as for NCCL). A barrier that waits longer than CEC_PEER_TIMEOUT_S
 * (environment, default 60 s) for a peer sets an error flag instead of hanging: the call returns
 * CEC_E_NCCL and the context stays in that state. The paper's SIMT engine keeps NCCL.
 * Errors: CEC_E_ARG (world outside 2..8, blob mismatch), CEC_E_CUDA (allocation / IPC failure, a
 * peer device not visible, or no native P2P atomics between this device and a peer: the caller then
 * keeps the NCCL path). */
#define CEC_PEER_BLOB_BYTES 128
cec_status cec_peer_export(cec_ctx *ctx, void *blob_out);
cec_status cec_peer_import(cec_ctx *ctx, const void *blobs);

/* Emulation of several ranks on ONE device (tests only; a one-GPU box has no second GPU). Kernels
 * that wait on one another must not run as separate launches on one GPU: nothing makes them
 * co-resident, and on B200 two or four such processes raised Xid 109 (context-switch timeout,
 * /opt/skills/guides/B200_PROFILING.md). With `fn` set, every peer barrier of a run becomes
 * "drain this rank's stream, then call fn(user)", where fn is the caller's host barrier across the
 * emulated ranks (e.g. a gloo dist.barrier()); no kernel ever waits for another rank, and runs are
 * not captured in CUDA graphs. Everything else of the peer path is unchanged (IPC mappings,
 * system-scope atomicMin into rank 0's home arrays, cross-rank bounds, gather). fn = NULL restores
 * the device barriers. Call after cec_peer_import, on every rank.
 * Errors: CEC_E_ARG (null ctx), CEC_E_STATE (the context is not in peer mode). */
cec_status cec_peer_host_barrier(cec_ctx *ctx, void (*fn)(void *user), void *user);

/* Host utility exported for tests: the contiguous slice range [*begin, *end) of `n` slices that
 * rank `rank` of `world` simulates (pattern-space sharding). */
void cec_shard_range(uint64_t n, int32_t rank, int32_t world, uint64_t *begin, uint64_t *end);
/* Host utility exported for tests: parallel bit extract (idx_own = pext(idx_merged, ownmask)). */
uint64_t cec_pext64(uint64_t value, uint64_t mask);

void cec_free(cec_ctx *ctx);
const char *cec_last_error(const cec_ctx *ctx);
int cec_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* CEC_H */
