// cec_ctx.hpp — the context and plan structures behind the opaque handles of include/cec.h,
// shared by the host driver translation units (cec_host.cpp, cuts.cpp). Not part of the ABI.
#pragma once
#include <nccl.h>

#include <algorithm>
#include <atomic>
#include <condition_variable>
#include <cstdint>
#include <cstdlib>
#include <functional>
#include <memory>
#include <mutex>
#include <thread>
#include <string>
#include <vector>

#include "../../include/cec.h"
#include "cec_internal.hpp"

using namespace cec;

// ------------------------------------------------------------------------------------------------
// Context and plan
// ------------------------------------------------------------------------------------------------
// Per-thread traversal scratch: epoch-stamped flat arrays over node ids (no hashing on the host
// hot path); one per planning thread.
struct Scratch {
    std::vector<uint32_t> stamp, stack;
    uint32_t epoch = 0;
    std::vector<uint32_t> sc_stamp, sc_pos, sc_last, sc_slot;
    uint32_t sc_epoch = 0;
    std::vector<uint32_t> stop;
    uint32_t stop_epoch = 0;
    void init(size_t N) {
        if (stamp.size() == N) return;
        stamp.assign(N, 0);
        sc_stamp.assign(N, 0);
        sc_pos.assign(N, 0);
        sc_last.assign(N, 0);
        sc_slot.assign(N, 0);
        stop.assign(N, 0);
        epoch = sc_epoch = stop_epoch = 0;
    }
    uint32_t next_epoch() {
        if (++epoch == 0) {
            std::fill(stamp.begin(), stamp.end(), 0u);
            epoch = 1;
        }
        return epoch;
    }
    uint32_t next_stop() {
        if (++stop_epoch == 0) {
            std::fill(stop.begin(), stop.end(), 0u);
            stop_epoch = 1;
        }
        return stop_epoch;
    }
};

// Persistent host worker pool of a context (planning, supports, JIT compiles, cut enumeration):
// threads are created once and sleep on a condition variable between jobs, so a call that plans
// many small batches (pipelined chunks, Alg. 2 buffer flushes) pays no thread start-up per batch.
// run(n, fn) calls fn(item, tid) for items 0..n-1; tid in [0, size()] (the caller is the last tid).
struct WorkPool {
    std::vector<std::thread> th;
    std::mutex mu;
    std::condition_variable cv, done_cv;
    std::atomic<uint64_t> gen{0};
    std::atomic<bool> quit{false};
    std::atomic<uint32_t> next{0}, busy{0};
    uint32_t n = 0;
    const std::function<void(uint32_t, unsigned)> *fn = nullptr;
    // run(..., spin = true): after that job the workers (and the caller waiting for them) spin
    // ~tens of microseconds before sleeping, so a loop of short jobs (Alg. 2 cut enumeration: one
    // job per enumeration level) starts each job without a futex wake-up of every worker. Other
    // callers keep spin off: spinning workers slow the caller's serial work between jobs (C3
    // planning 2% slower with spinning everywhere). CEC_POOL_SPIN = pause iterations (4096).
    const int kSpin = getenv("CEC_POOL_SPIN") ? atoi(getenv("CEC_POOL_SPIN")) : 4096;
    std::atomic<int> spin_now{0};  // spin budget of the current job
    static inline void relax() {
#if defined(__x86_64__) || defined(__i386__)
        __builtin_ia32_pause();
#endif
    }
    explicit WorkPool(unsigned workers) {
        for (unsigned t = 0; t < workers; ++t) th.emplace_back([this, t]() { loop(t); });
    }
    unsigned size() const { return (unsigned)th.size(); }
    void loop(unsigned tid) {
        uint64_t seen = 0;
        int budget = 0;
        for (;;) {
            int i = 0;
            while (i < budget && gen.load(std::memory_order_acquire) == seen && !quit.load(std::memory_order_relaxed)) {
                relax();
                ++i;
            }
            if (i >= budget && gen.load(std::memory_order_acquire) == seen) {
                std::unique_lock<std::mutex> l(mu);
                cv.wait(l, [&]() { return quit.load() || gen.load(std::memory_order_acquire) != seen; });
            }
            if (quit.load()) return;
            seen = gen.load(std::memory_order_acquire);
            budget = spin_now.load(std::memory_order_relaxed);
            work(tid);
            if (busy.fetch_sub(1, std::memory_order_acq_rel) == 1) {
                std::lock_guard<std::mutex> l(mu);
                done_cv.notify_all();
            }
        }
    }
    void work(unsigned tid) {
        for (uint32_t i; (i = next.fetch_add(1, std::memory_order_relaxed)) < n;) (*fn)(i, tid);
    }
    void run(uint32_t items, const std::function<void(uint32_t, unsigned)> &f, bool spin = false) {
        if (th.empty() || items < 2) {
            for (uint32_t i = 0; i < items; ++i) f(i, size());
            return;
        }
        {
            std::lock_guard<std::mutex> l(mu);
            fn = &f;
            n = items;
            next.store(0, std::memory_order_relaxed);
            busy.store(size(), std::memory_order_relaxed);
            spin_now.store(spin ? kSpin : 0, std::memory_order_relaxed);
            gen.fetch_add(1, std::memory_order_release);  // publishes fn / n / next / busy / spin
        }
        cv.notify_all();
        work(size());
        for (int i = 0; spin && i < kSpin && busy.load(std::memory_order_acquire) != 0; ++i) relax();
        if (busy.load(std::memory_order_acquire) != 0) {
            std::unique_lock<std::mutex> l(mu);
            done_cv.wait(l, [&]() { return busy.load(std::memory_order_acquire) == 0; });
        }
    }
    ~WorkPool() {
        {
            std::lock_guard<std::mutex> l(mu);
            quit.store(true);
        }
        cv.notify_all();
        for (auto &t : th) t.join();
    }
};

struct cec_ctx {
    uint32_t I = 0, A = 0, O = 0;
    std::vector<uint32_t> f0, f1;  // fanin literals indexed by node id (valid for AND ids)
    std::vector<uint32_t> level;   // a1: level(PI)=0, level(AND)=1+max(fanins)
    cec_opts opts{};
    bool host_only = true;
    void *stream = nullptr, *own_stream = nullptr;
    AuxStreams aux;  // side streams for concurrent launch groups
    int num_sms = 0;
    ncclComm_t comm = nullptr;
    PeerState peer;  // a10 over NVLink peer memory (peer.cu), set up by cec_peer_export/import
    std::string err;
    cec_stats stats{};
    // last global check (for cec_get_cex)
    bool have_last = false;
    std::vector<int32_t> last_verdict;
    std::vector<uint64_t> last_cex;
    std::vector<std::vector<uint32_t>> last_support;
    // device copy of the AIG for random simulation (lazy)
    uint32_t *d_f0 = nullptr, *d_f1 = nullptr, *d_level_ids = nullptr;
    uint64_t d_aig_cap = 0;     // entries allocated in each of d_f0 / d_f1 / d_level_ids
    bool d_aig_valid = false;   // they hold THIS AIG (cec_reload_aig keeps the buffers, not the data)
    NodeSupports supp_table;  // a2 per-node support lists on the device (AIG-only, built once)
    std::vector<uint32_t> level_off;
    std::shared_ptr<DevPool> devpool;  // plan device blocks + pinned staging (device contexts)
    Scratch scratch;  // for serial host work (supports of single pairs, cut validation)
    std::vector<Scratch> pool;  // one per planning thread, kept across calls (allocated once)
    std::unique_ptr<WorkPool> wpool;  // persistent host workers (lazy)
    WorkPool &workers() {
        if (!wpool) {
            const unsigned hw = std::max(1u, std::min(32u, std::thread::hardware_concurrency()));
            wpool.reset(new WorkPool(hw - 1));
            if (pool.size() < hw) pool.resize(hw);
        }
        return *wpool;
    }

    uint32_t N() const { return 1 + I + A; }
    bool is_and(uint32_t id) const { return id > I; }
};

// std::allocator that default-initialises (no zero fill on resize): the interpreter programs of a
// plan (~9 MB for C3) are resized and then fully overwritten by a parallel copy.
template <class T>
struct DefaultInitAlloc : std::allocator<T> {
    template <class U>
    struct rebind {
        using other = DefaultInitAlloc<U>;
    };
    DefaultInitAlloc() = default;
    template <class U>
    DefaultInitAlloc(const DefaultInitAlloc<U> &) noexcept {}
    template <class U>
    void construct(U *p) noexcept {
        ::new (static_cast<void *>(p)) U;
    }
    template <class U, class... A>
    void construct(U *p, A &&...a) {
        ::new (static_cast<void *>(p)) U(std::forward<A>(a)...);
    }
};

struct WinHost {
    std::vector<uint32_t> inputs;  // node ids, increasing
    std::vector<uint32_t> cmps;    // compare indices of this window
    uint64_t est_nodes = 0;        // cone-size estimate used by the cost-aware merge
};

struct Cmp {
    uint32_t la, lb;
    uint64_t ownmask = 0;          // bit j set if window input j belongs to this pair's own support
    std::vector<uint32_t> S;       // own inputs (global: support; local: leaves)
};

struct cec_plan {
    ~cec_plan();  // returns the device block (cec_host.cpp)
    bool local = false;
    uint32_t num_pairs = 0;
    std::vector<uint32_t> la, lb;      // the caller's pairs
    std::vector<int32_t> pre_verdict;  // per user pair: -100 = decided by simulation
    std::vector<uint64_t> pre_cex;
    std::vector<uint32_t> k;
    std::vector<int32_t> pair_cmp;
    std::vector<Cmp> cmps;
    // windows after merging
    std::vector<std::vector<uint32_t>> win_inputs;
    std::vector<uint32_t> win_nodes;          // AND-node count per window
    std::vector<std::vector<uint32_t>> win_cmps;
    std::vector<DevWin> dwin;
    std::vector<uint4, DefaultInitAlloc<uint4>> prog;  // every slot written by finish_plan
    std::vector<Item> items;
    std::vector<JItem> jitems;
    std::vector<uint32_t> joff;  // free-warp groups' per-warp item offsets (relative to the group)
    std::vector<LaunchGroup> groups;
    uint32_t jit_windows = 0, jit_kernels = 0;
    float jit_ms = 0.f;
    uint64_t lop3_words = 0;
    uint64_t imad_words = 0;  // IMAD cells x words (JIT mode 3)
    SimtPlan simt;  // CEC_ENGINE_SIMT plans
    uint64_t W_rank = 0, W_all = 0;
    uint32_t max_k = 0, max_slots = 0;
    float host_ms = 0.f;
    // device
    bool uploaded = false;
    DevPlan d;
    std::shared_ptr<DevPool> pool;  // owner of the block below
    void *arena = nullptr;          // one device block holding every DevPlan buffer
    size_t arena_cap = 0;
    void *ev0 = nullptr, *ev1 = nullptr;
    void *sev[2] = {nullptr, nullptr};  // around the window kernels only (launch_run sweep_ev)
    bool sweep_timing = false;           // record sev in runs (cec_plan_sweep_timing; off: no cost)
    bool sweep_timed_last = false;       // the last run recorded sev
    bool ran = false;
    bool no_join = false;  // pipelined call, not its last chunk: skip the side-stream join (launch_run)
    uint32_t runs = 0;                     // completed cec_plan_run calls
    void *graph = nullptr, *graph_stream = nullptr;  // captured run (replayed from the 2nd run on)
    uint32_t graph_launches = 0;
    uint32_t graph_peer_gen = 0;  // PeerState::gen the graph was captured with
};


// a12 in two steps (cec_host.cpp): validate + plan + upload + launch asynchronously, then collect
cec_status local_checks_launch(cec_ctx *c, uint32_t n, const uint32_t *la, const uint32_t *lb, const uint32_t *cut_off,
                               const uint32_t *leaves, std::unique_ptr<cec_plan> &out, uint32_t *bad_out,
                               uint32_t *first_bad_out, bool trusted_cuts = false);
cec_status local_checks_collect(cec_ctx *c, cec_plan *P, int32_t *verdict);

// device copy of the AIG (fanin literals + level CSR), uploaded on first use (cec_host.cpp)
extern "C" cec_status cec_ensure_device_aig(cec_ctx *c);  // internal (not in include/cec.h)
