// sim_interp.cu — sm_100a schedule-interpreter kernel for exhaustive bit-parallel simulation.
//
// What it computes (§III-B, Alg. 1 reconstructed in SURVEY.md App. A): for every
// window, every u32 word w of the 2^k-pattern truth table of every window node, with the input
// (projection) words generated arithmetically, AND nodes evaluated in topological
// order, and every candidate pair XOR-compared; the minimum mismatching pattern index per pair is
// recorded with atomicMin (canonical CEX).
//
// B200 design (differs from the paper's Alg. 1):
//  * no simulation table in HBM: each warp owns a 32-word slice of the pattern space and carries it
//    through the whole window; node words live in shared-memory slots [slot][lane] allocated by
//    liveness on the host, so a window's working set is (live nodes) x 128 B per warp;
//  * levels are program order inside a warp (no grid-wide level barrier, no per-level launch);
//  * windows and slices are work items pulled by warps from a global counter (dims 2 and 3 of
//    PAPER.md:114-116 folded into one dynamic queue, largest windows first);
//  * compare ops are interleaved right after the later root is computed; __ballot_sync finds the
//    lowest mismatching lane (= lowest word), __ffs the lowest bit; a window whose pairs are all
//    refuted publishes a bound and later slices above it are skipped (bounded early exit, Q9).
#include <cuda_runtime.h>
#include <chrono>

#include <cstdio>
#include <cstdlib>

#include <algorithm>
#include <cstdint>
#include <vector>

#include "cec_internal.hpp"

namespace cec {

namespace {

constexpr uint32_t FULL = 0xFFFFFFFFu;
constexpr int MAX_WPB = 4;  // warps per block
constexpr size_t SMEM_PER_SM = 227 * 1024;

__device__ __forceinline__ uint32_t proj_word(uint32_t j, uint64_t w) {
    // projection truth table of input j at word w: bit b of word w is pattern
    // i = 32 w + b, and input j takes bit j of i.
    switch (j) {
        case 0: return 0xAAAAAAAAu;
        case 1: return 0xCCCCCCCCu;
        case 2: return 0xF0F0F0F0u;
        case 3: return 0xFF00FF00u;
        case 4: return 0xFFFF0000u;
        default: return 0u - (uint32_t)((w >> (j - 5)) & 1u);
    }
}

__device__ __forceinline__ uint32_t lop3_60(uint32_t t, uint32_t b, uint32_t m) {
    uint32_t r;
    asm("lop3.b32 %0, %1, %2, %3, 0x60;" : "=r"(r) : "r"(t), "r"(b), "r"(m));
    return r;
}

__device__ __noinline__ void record_mismatch(uint32_t c, uint64_t idx, uint32_t win, const DevWin &W,
                                             unsigned long long *first, unsigned long long *bound,
                                             uint32_t *neq_cnt) {
    // system scope: in peer mode (peer.cu) these arrays are rank 0's, written by every GPU
    unsigned long long old = atomicMin_system(&first[c], (unsigned long long)idx);
    if (old == ~0ull) {
        __threadfence_system();
        uint32_t n = atomicAdd_system(&neq_cnt[win], 1u) + 1u;
        if (n == W.ncmp) {  // every pair of the window is refuted: publish an early-exit bound
            __threadfence_system();
            unsigned long long mx = 0;
            for (uint32_t t = 0; t < W.ncmp; ++t) {
                unsigned long long v = atomicAdd_system(&first[W.cmp_off + t], 0ull);
                mx = v > mx ? v : mx;
            }
            atomicMin_system(&bound[win], mx);
        }
    }
}

__device__ __forceinline__ void report(uint32_t d, uint64_t word_base, uint32_t lane, uint32_t c, uint32_t win,
                                       const DevWin &W, unsigned long long *first, unsigned long long *bound,
                                       uint32_t *neq_cnt) {
    // d = this lane's mismatch bits for word word_base + lane (all lanes of the warp call this)
    const uint32_t bal = __ballot_sync(FULL, d != 0u);
    const uint32_t l = (uint32_t)__ffs(bal) - 1u;
    const uint32_t dl = __shfl_sync(FULL, d, l);
    if (lane == 0) record_mismatch(c, ((word_base + l) << 5) + (uint32_t)(__ffs(dl) - 1), win, W, first, bound, neq_cnt);
}

// One warp = one slice of 32*IV consecutive words: lane l holds words base + v*32 + l (v < IV), so
// a ballot over v = 0 before v = 1 finds mismatches in pattern order.
__global__ void __launch_bounds__(MAX_WPB * 32)
interp_kernel(const Item *__restrict__ items, uint32_t nitems, uint32_t *__restrict__ item_ctr,
              const DevWin *__restrict__ wins, const uint4 *__restrict__ prog, unsigned long long *first,
              unsigned long long *bound, uint32_t *neq_cnt, uint32_t nslots) {
    extern __shared__ __align__(16) unsigned char smem[];
    const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31u;
    unsigned char *wbase = smem + (size_t)warp * (nslots * SLOT_BYTES + 32u * sizeof(uint4));
    uint4 *ibuf = reinterpret_cast<uint4 *>(wbase + nslots * SLOT_BYTES);
    unsigned char *my = wbase + lane * (IV * 4u);  // this lane's uint2 inside every slot
#define SLOT(off) (*reinterpret_cast<uint2 *>(my + (off)))

    for (;;) {
        uint32_t it = 0;
        if (lane == 0) it = atomicAdd(item_ctr, 1u);
        it = __shfl_sync(FULL, it, 0);
        if (it >= nitems) break;
        const Item item = items[it];
        const DevWin W = wins[item.win];
        const uint64_t tt_words = ((uint64_t)W.tt_words_hi << 32) | W.tt_words_lo;
        for (uint32_t s = item.s_begin; s < item.s_end; ++s) {
            const uint64_t base = (uint64_t)s * (32u * IV);  // first word of the slice
            // bounded early exit (Q9): lane 0 reads the window bound and the warp takes ITS value,
            // so the break and the full-mask votes below stay warp-uniform
            unsigned long long bw = 0ull;
            if (lane == 0) bw = *((volatile unsigned long long *)&bound[item.win]);
            if ((base << 5) >= __shfl_sync(FULL, bw, 0)) break;
            const uint64_t w0 = base + lane, w1 = base + 32u + lane;
            const bool act0 = w0 < tt_words, act1 = w1 < tt_words;
            for (uint32_t j = 0; j < W.k; ++j) SLOT(j * SLOT_BYTES) = make_uint2(proj_word(j, w0), proj_word(j, w1));
            if (W.const_slot != 0xFFFFFFFFu) SLOT(W.const_slot * SLOT_BYTES) = make_uint2(0u, 0u);
            for (uint32_t p = 0; p < W.prog_len; p += 32u) {
                const uint32_t n = min(32u, W.prog_len - p);
                __syncwarp();
                if (lane < n) ibuf[lane] = prog[W.prog_off + p + lane];
                __syncwarp();
#pragma unroll 4
                for (uint32_t j = 0; j < n; ++j) {
                    const uint4 ins = ibuf[j];
                    const uint32_t ma = (uint32_t)((int32_t)(ins.x << 31) >> 31);
                    const uint32_t mb = (uint32_t)((int32_t)(ins.y << 31) >> 31);
                    const uint2 a = SLOT(ins.x & ~7u), b = SLOT(ins.y & ~7u);
                    const uint32_t a0 = a.x ^ ma, a1 = a.y ^ ma;
                    if (!(ins.z & OP_CMP)) {
                        // (a ^ ma) & (b ^ mb) as one LOP3 per word on the pre-complemented a:
                        // inputs (t, b, m) = (0xF0, 0xCC, 0xAA): t & (b ^ m) = 0x60
                        SLOT(ins.z) = make_uint2(lop3_60(a0, b.x, mb), lop3_60(a1, b.y, mb));
                    } else {
                        const uint32_t d0 = act0 ? (a0 ^ b.x ^ mb) : 0u, d1 = act1 ? (a1 ^ b.y ^ mb) : 0u;
                        if (__any_sync(FULL, (d0 | d1) != 0u)) {
                            if (__any_sync(FULL, d0 != 0u))
                                report(d0, base, lane, ins.z & ~OP_CMP, item.win, W, first, bound, neq_cnt);
                            else
                                report(d1, base + 32u, lane, ins.z & ~OP_CMP, item.win, W, first, bound, neq_cnt);
                        }
                    }
                }
            }
        }
    }
#undef SLOT
}

inline const char *ck(cudaError_t e) { return e == cudaSuccess ? nullptr : cudaGetErrorString(e); }

__global__ void reset_run(unsigned long long *first, uint32_t ncmp, unsigned long long *bound, uint32_t *neq_cnt,
                          uint32_t nwin, uint32_t *item_ctr, uint32_t ngroups) {
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < ncmp) first[i] = ~0ull;
    if (i < nwin) {
        bound[i] = ~0ull;
        neq_cnt[i] = 0u;
    }
    if (i < ngroups) item_ctr[i] = 0u;
}

}  // namespace

uint32_t interp_max_slots_per_warp() {
    // one warp per block, whole shared memory: nslots * SLOT_BYTES + 512 <= 227 KB
    return (uint32_t)((SMEM_PER_SM - 32 * sizeof(uint4)) / SLOT_BYTES);
}

const char *aux_create(AuxStreams &a) {
    if (a.ok) return nullptr;
    const char *e;
    a.n = 4;
    if (const char *v = getenv("CEC_SIDE_STREAMS")) a.n = std::max(1, std::min(NAUX_MAX, atoi(v)));
    for (int i = 0; i < a.n; ++i) {
        cudaStream_t s;
        if ((e = ck(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking)))) return e;
        a.s[i] = s;
        cudaEvent_t ev;
        if ((e = ck(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming)))) return e;
        a.join[i] = ev;
    }
    cudaEvent_t f;
    if ((e = ck(cudaEventCreateWithFlags(&f, cudaEventDisableTiming)))) return e;
    a.fork = f;
    a.ok = true;
    return nullptr;
}

void aux_destroy(AuxStreams &a) {
    for (int i = 0; i < a.n; ++i) {
        if (a.s[i]) cudaStreamDestroy((cudaStream_t)a.s[i]);
        if (a.join[i]) cudaEventDestroy((cudaEvent_t)a.join[i]);
    }
    if (a.fork) cudaEventDestroy((cudaEvent_t)a.fork);
    a = AuxStreams{};
}

// event record that also works inside a stream capture (as an external event-record node)
static const char *record_span_event(void *ev, cudaStream_t st) {
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    const char *e = ck(cudaStreamIsCapturing(st, &cs));
    if (e) return e;
    return ck(cs == cudaStreamCaptureStatusActive
                  ? cudaEventRecordWithFlags((cudaEvent_t)ev, st, cudaEventRecordExternal)
                  : cudaEventRecord((cudaEvent_t)ev, st));
}

const char *launch_run(const DevPlan &d0, const std::vector<LaunchGroup> &groups, uint32_t nwin, uint32_t ncmp,
                       void *stream, int num_sms, uint32_t *launches, AuxStreams *aux, const PeerRun *pr,
                       bool no_join, void *const *sweep_ev) {
    cudaStream_t main_st = (cudaStream_t)stream;
    cudaStream_t st = main_st;
    const char *e;
    const bool peer = pr && pr->on;
    DevPlan d = d0;
    if (peer) {  // the window kernels update rank 0's home arrays directly (peer.cu)
        d.first = pr->home_first;
        d.bound = pr->home_bound;
        d.neq_cnt = pr->home_neq;
    }
    {  // one launch resets the run state (first-mismatch indices, bounds, counters); in peer mode
       // only rank 0 resets the home arrays, every rank its own item counters
        const uint32_t ng = (uint32_t)(groups.size() ? groups.size() : 1);
        const uint32_t rc = peer && pr->rank != 0 ? 0u : ncmp, rw = peer && pr->rank != 0 ? 0u : nwin;
        const uint32_t n = std::max(std::max(rc, rw), ng);
        reset_run<<<(n + 255) / 256, 256, 0, st>>>(d.first, rc, d.bound, d.neq_cnt, rw, d.item_ctr, ng);
        if ((e = ck(cudaGetLastError()))) return e;
    }
    uint32_t nl = 0;
    if (peer) {  // home reset on rank 0 before any rank's kernels touch it
        if ((e = peer_barrier_launch(*pr, main_st))) return e;
        ++nl;
    }
    const bool multi = aux && aux->ok && groups.size() > 1 && getenv("CEC_PROFILE_GROUPS") == nullptr;
    const bool span = sweep_ev && sweep_ev[0] && sweep_ev[1] && !(multi && no_join);
    if (span && (e = record_span_event(sweep_ev[0], main_st))) return e;
    if (multi) {
        if ((e = ck(cudaEventRecord((cudaEvent_t)aux->fork, main_st)))) return e;
        for (int i = 0; i < aux->n; ++i)
            if ((e = ck(cudaStreamWaitEvent((cudaStream_t)aux->s[i], (cudaEvent_t)aux->fork, 0)))) return e;
    }
    // CEC_PROFILE_GROUPS=1: serial launches, each group timed with events, one line per group on stderr
    static const bool prof = getenv("CEC_PROFILE_GROUPS") != nullptr;
    std::vector<cudaEvent_t> pev;
    if (prof && !multi) {
        pev.resize(groups.size() + 1);
        for (auto &x : pev) cudaEventCreate(&x);
        cudaEventRecord(pev[0], main_st);
    }
    // CEC_TIMING=2: host time of each launch (stderr)
    static const bool lt = getenv("CEC_TIMING") && atoi(getenv("CEC_TIMING")) >= 2;
    auto lnow = []() { return std::chrono::steady_clock::now(); };
    auto lt0 = lnow();
    for (size_t g = 0; g < groups.size(); ++g) {
        const LaunchGroup &G = groups[g];
        if (lt && g > 0) {
            const auto t = lnow();
            fprintf(stderr, "[cec]   launch group %zu (%s): %.3f ms host\n", g - 1, groups[g - 1].jit ? "jit" : "interp",
                    std::chrono::duration<double, std::milli>(t - lt0).count());
            lt0 = t;
        }
        if (!pev.empty() && g > 0) cudaEventRecord(pev[g], main_st);
        if (G.nitems == 0) continue;
        // the biggest group stays on the caller's stream; the others round-robin on side streams
        st = (multi && g > 0) ? (cudaStream_t)aux->s[(g - 1) % aux->n] : main_st;
        stream = st;
        if (G.jit) {
            // a free-warp kernel reads its per-warp item offsets where the others take their counter
            uint32_t *ctr = G.free_blocks ? d.joff + G.joff_off : d.item_ctr + g;
            if ((e = jit_launch(G.jit, d.jitems + G.item_off, G.nitems, ctr, d.first, d.bound, d.neq_cnt,
                                stream, num_sms, G.free_blocks)))
                return e;
            ++nl;
            continue;
        }
        const size_t per_warp = (size_t)G.nslots * SLOT_BYTES + 32 * sizeof(uint4);
        // warps per block: the choice that keeps the most warps resident per SM (smem-limited)
        int wpb = 1;
        size_t best = 0;
        for (int w = MAX_WPB; w >= 1; w >>= 1) {
            const size_t per_block = per_warp * w + 1024;  // + per-block reservation
            const size_t resident = (size_t)w * std::min<size_t>(32 / w, (SMEM_PER_SM + 1024) / per_block);
            if (resident > best) {
                best = resident;
                wpb = w;
            }
        }
        const size_t smem = per_warp * wpb;
        if (smem > SMEM_PER_SM) return "window live set exceeds shared memory";
        if ((e = ck(cudaFuncSetAttribute(interp_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem))))
            return e;
        int per_sm = 0;
        if ((e = ck(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, interp_kernel, wpb * 32, smem)))) return e;
        if (per_sm < 1) per_sm = 1;
        uint64_t grid = (uint64_t)num_sms * per_sm;
        const uint64_t need = (G.nitems + wpb - 1) / wpb;
        if (grid > need) grid = need;
        interp_kernel<<<(unsigned)grid, wpb * 32, smem, st>>>(d.items + G.item_off, G.nitems, d.item_ctr + g, d.wins,
                                                              d.prog, d.first, d.bound, d.neq_cnt, G.nslots);
        if ((e = ck(cudaGetLastError()))) return e;
        ++nl;
    }
    if (!pev.empty()) {
        cudaEventRecord(pev[groups.size()], main_st);
        cudaEventSynchronize(pev[groups.size()]);
        for (size_t g = 0; g < groups.size(); ++g) {
            float ms = 0.f;
            cudaEventElapsedTime(&ms, pev[g], pev[g + 1]);
            const LaunchGroup &G = groups[g];
            fprintf(stderr, "group %zu %s win=%u max_k=%u nodes=%u items=%u lop3_words=%llu ms=%.4f tlop3=%.3f\n", g,
                    G.jit ? "jit" : "interp", G.nwin, G.max_k, G.nodes, G.nitems, (unsigned long long)G.lop3_words,
                    ms, ms > 0 ? G.lop3_words / (ms * 1e9) : 0.0);
        }
        for (auto &x : pev) cudaEventDestroy(x);
    }
    if (multi && !(no_join && !peer)) {  // join: the caller's stream waits for every side stream
        for (int i = 0; i < aux->n; ++i) {
            if ((e = ck(cudaEventRecord((cudaEvent_t)aux->join[i], (cudaStream_t)aux->s[i])))) return e;
            if ((e = ck(cudaStreamWaitEvent(main_st, (cudaEvent_t)aux->join[i], 0)))) return e;
        }
    }
    if (span && (e = record_span_event(sweep_ev[1], main_st))) return e;
    if (peer) {  // every rank's kernels done -> gather the minimum -> nobody resets before all gathered
        if ((e = peer_barrier_launch(*pr, main_st))) return e;
        if ((e = peer_gather_launch(*pr, ncmp, main_st))) return e;
        if ((e = peer_barrier_launch(*pr, main_st))) return e;
        nl += ncmp ? 3 : 2;
    }
    if (launches) *launches = nl;
    return nullptr;
}

// CUDA graph of one plan run (the reset kernel plus every window launch with its side-stream
// fork/join): captured once per (plan, stream) and replayed, so a re-run costs one graph launch
// instead of one host launch per group (C3: ~1.6k launches per run).
const char *graph_capture_run(const DevPlan &d, const std::vector<LaunchGroup> &groups, uint32_t nwin, uint32_t ncmp,
                              void *stream, int num_sms, uint32_t *launches, AuxStreams *aux, void **exec_out,
                              const PeerRun *pr, void *const *sweep_ev) {
    cudaStream_t st = (cudaStream_t)stream;
    const char *e;
    *exec_out = nullptr;
    if ((e = ck(cudaStreamBeginCapture(st, cudaStreamCaptureModeRelaxed)))) return e;
    const char *le = launch_run(d, groups, nwin, ncmp, stream, num_sms, launches, aux, pr, false, sweep_ev);
    cudaGraph_t g = nullptr;
    const char *ee = ck(cudaStreamEndCapture(st, &g));
    if (le || ee) {
        if (g) cudaGraphDestroy(g);
        return le ? le : ee;
    }
    cudaGraphExec_t x = nullptr;
    e = ck(cudaGraphInstantiate(&x, g, 0));
    cudaGraphDestroy(g);
    if (e) return e;
    *exec_out = x;
    return nullptr;
}
const char *graph_launch(void *exec, void *stream) {
    return ck(cudaGraphLaunch((cudaGraphExec_t)exec, (cudaStream_t)stream));
}
void graph_destroy(void *exec) {
    if (exec) cudaGraphExecDestroy((cudaGraphExec_t)exec);
}

const char *DevPool::get(size_t bytes, void **p, size_t *cap) {
    {
        std::lock_guard<std::mutex> g(mu);
        size_t best = free_blocks.size();
        for (size_t i = 0; i < free_blocks.size(); ++i)
            if (free_blocks[i].second >= bytes && (best == free_blocks.size() || free_blocks[i].second < free_blocks[best].second))
                best = i;
        if (best < free_blocks.size()) {
            *p = free_blocks[best].first;
            *cap = free_blocks[best].second;
            free_blocks.erase(free_blocks.begin() + best);
            return nullptr;
        }
    }
    const size_t c = (std::max<size_t>(bytes, 1) + (2u << 20) - 1) / (2u << 20) * (2u << 20);
    const char *e = ck(cudaMalloc(p, c));
    *cap = e ? 0 : c;
    return e;
}
void DevPool::put(void *p, size_t cap) {
    if (!p) return;
    std::lock_guard<std::mutex> g(mu);
    free_blocks.emplace_back(p, cap);
    size_t total = 0;
    for (auto &b : free_blocks) total += b.second;
    while (total > (1ull << 30) && free_blocks.size() > 1) {  // keep at most ~1 GiB cached
        auto it = std::max_element(free_blocks.begin(), free_blocks.end(),
                                   [](const std::pair<void *, size_t> &a, const std::pair<void *, size_t> &b) {
                                       return a.second < b.second;
                                   });
        total -= it->second;
        cudaFree(it->first);
        free_blocks.erase(it);
    }
}
const char *DevPool::staging(size_t bytes, void **host) {
    const char *e;
    if (pinned_ev && (e = ck(cudaEventSynchronize((cudaEvent_t)pinned_ev)))) return e;
    if (bytes > pinned_bytes) {
        if (pinned) cudaFreeHost(pinned);
        pinned = nullptr;
        const size_t c = (bytes + (1u << 20) - 1) / (1u << 20) * (1u << 20);
        if ((e = ck(cudaMallocHost(&pinned, c)))) {
            pinned_bytes = 0;
            return e;
        }
        pinned_bytes = c;
    }
    *host = pinned;
    return nullptr;
}
const char *DevPool::staged(void *stream) {
    const char *e;
    if (!pinned_ev) {
        cudaEvent_t ev;
        if ((e = ck(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming)))) return e;
        pinned_ev = ev;
    }
    return ck(cudaEventRecord((cudaEvent_t)pinned_ev, (cudaStream_t)stream));
}
DevPool::~DevPool() {
    if (pinned_ev) {
        cudaEventSynchronize((cudaEvent_t)pinned_ev);
        cudaEventDestroy((cudaEvent_t)pinned_ev);
    }
    if (pinned) cudaFreeHost(pinned);
    for (auto &b : free_blocks) cudaFree(b.first);
}

const char *dev_alloc(void **p, size_t bytes) { return ck(cudaMalloc(p, bytes ? bytes : 16)); }
const char *dev_free(void *p) { return p ? ck(cudaFree(p)) : nullptr; }
const char *h2d(void *dst, const void *src, size_t bytes, void *stream) {
    return bytes ? ck(cudaMemcpyAsync(dst, src, bytes, cudaMemcpyHostToDevice, (cudaStream_t)stream)) : nullptr;
}
const char *d2h(void *dst, const void *src, size_t bytes, void *stream) {
    return bytes ? ck(cudaMemcpyAsync(dst, src, bytes, cudaMemcpyDeviceToHost, (cudaStream_t)stream)) : nullptr;
}
const char *dev_memset(void *dst, int v, size_t bytes, void *stream) {
    return bytes ? ck(cudaMemsetAsync(dst, v, bytes, (cudaStream_t)stream)) : nullptr;
}
const char *stream_sync(void *stream) { return ck(cudaStreamSynchronize((cudaStream_t)stream)); }
const char *dev_init(int device, void **own_stream, int *num_sms) {
    int n = 0;
    const char *e;
    if ((e = ck(cudaGetDeviceCount(&n)))) return e;
    if (device < 0 || device >= n) return "no such CUDA device";
    if ((e = ck(cudaSetDevice(device)))) return e;
    cudaDeviceProp prop;
    if ((e = ck(cudaGetDeviceProperties(&prop, device)))) return e;
    if (prop.major != 10) return "libcec is built for sm_100a (B200); this device is not compute capability 10.x";
    *num_sms = prop.multiProcessorCount;
    cudaStream_t s;
    if ((e = ck(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking)))) return e;
    *own_stream = s;
    return nullptr;
}
const char *stream_destroy(void *stream) { return stream ? ck(cudaStreamDestroy((cudaStream_t)stream)) : nullptr; }
const char *event_create(void **ev) {
    cudaEvent_t e;
    const char *r = ck(cudaEventCreate(&e));
    *ev = r ? nullptr : e;
    return r;
}
const char *event_record(void *ev, void *stream) { return ck(cudaEventRecord((cudaEvent_t)ev, (cudaStream_t)stream)); }
const char *event_elapsed(float *ms, void *a, void *b) {
    return ck(cudaEventElapsedTime(ms, (cudaEvent_t)a, (cudaEvent_t)b));
}
void event_destroy(void *ev) {
    if (ev) cudaEventDestroy((cudaEvent_t)ev);
}

}  // namespace cec
