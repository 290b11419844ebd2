// cec_host.cpp — host driver behind include/cec.h: AIG ingest and validation, structural supports,
// pair routing by support size, window construction and merging, liveness-allocated schedules,
// pattern-space sharding across ranks, NCCL min-reduction and result decoding.
//
// Paper map (PAPER.md line numbers):
//   a1 ingest/levels ........ :23, :27          a2 supports ............ :23, :81
//   a3 routing by k ......... :181, :183, :195  a4 windows ............. :81, :83, :114
//   a5 window merging ....... :120-124          a6 rounds -> pattern slices (:99, :118)
//   a9 compare / CEX ........ :57, :104-108     a10 cross-GPU min ...... north star (4)
//   a11 verdict + pext ...... :57, :69, :81     a12 local cuts ......... :128-130
#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <cstdarg>
#include <cstdlib>
#include <cstdio>
#include <cmath>
#include <cstring>
#include <map>
#include <memory>
#include <new>
#include <string>
#include <thread>
#include <unordered_map>
#include <vector>

#include "../../include/cec.h"
#include "cec_ctx.hpp"
#include "cec_internal.hpp"

using namespace cec;

// ------------------------------------------------------------------------------------------------
// NCCL, loaded on demand (world > 1 only) so the library loads on machines without it.
// ------------------------------------------------------------------------------------------------
namespace {
struct NcclApi {
    void *h = nullptr;
    ncclResult_t (*init_rank)(ncclComm_t *, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*all_reduce)(const void *, void *, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                               cudaStream_t) = nullptr;
    ncclResult_t (*destroy)(ncclComm_t) = nullptr;
    const char *(*err)(ncclResult_t) = nullptr;
    ncclResult_t (*get_id)(ncclUniqueId *) = nullptr;
    bool load() {
        if (h) return true;
        const char *names[] = {"libnccl.so.2", "libnccl.so"};
        for (const char *n : names) {
            h = dlopen(n, RTLD_NOW | RTLD_GLOBAL);
            if (h) break;
        }
        if (!h) return false;
        init_rank = (decltype(init_rank))dlsym(h, "ncclCommInitRank");
        all_reduce = (decltype(all_reduce))dlsym(h, "ncclAllReduce");
        destroy = (decltype(destroy))dlsym(h, "ncclCommDestroy");
        err = (decltype(err))dlsym(h, "ncclGetErrorString");
        get_id = (decltype(get_id))dlsym(h, "ncclGetUniqueId");
        return init_rank && all_reduce && destroy && err && get_id;
    }
};
NcclApi g_nccl;
}  // namespace

namespace {

thread_local std::string g_load_err;

cec_status fail(cec_ctx *c, cec_status s, const char *fmt, ...) {
    if (!c) {
        char buf[512];
        va_list ap;
        va_start(ap, fmt);
        vsnprintf(buf, sizeof buf, fmt, ap);
        va_end(ap);
        g_load_err = buf;
    } else {
        char buf[512];
        va_list ap;
        va_start(ap, fmt);
        vsnprintf(buf, sizeof buf, fmt, ap);
        va_end(ap);
        c->err = buf;
    }
    return s;
}

#define CUDA_TRY(ctx, expr)                                                         \
    do {                                                                            \
        const char *e_ = (expr);                                                    \
        if (e_) return fail((ctx), CEC_E_CUDA, "CUDA: %s (%s)", e_, #expr);          \
    } while (0)

// peer mode: did one of this rank's barriers time out (peer.cu)? Called after a stream sync.
static bool peer_failed(cec_ctx *c) {
    if (!c->peer.on) return false;
    bool t = false;
    return peer_error(c->peer, c->stream, &t) != nullptr || t;
}

// Structural TFI of the roots, stopping at nodes with stop_stamp == stop_epoch
// (cut leaves) and at PIs/const. Visits every reached node once; calls f(id) for each.
template <class F>
void walk_tfi(const cec_ctx *c, Scratch &X, const uint32_t *roots, int nroots, const std::vector<uint32_t> *stop,
              uint32_t stop_epoch, F &&f) {
    X.init(c->N());
    const uint32_t ep = X.next_epoch();
    auto &st = X.stack;
    auto &stamp = X.stamp;
    st.clear();
    for (int r = 0; r < nroots; ++r) {
        uint32_t v = roots[r];
        if (stamp[v] != ep) {
            stamp[v] = ep;
            st.push_back(v);
        }
    }
    while (!st.empty()) {
        uint32_t v = st.back();
        st.pop_back();
        f(v);
        if (stop && (*stop)[v] == stop_epoch) continue;
        if (!c->is_and(v)) continue;
        uint32_t a = c->f0[v] >> 1, b = c->f1[v] >> 1;
        if (stamp[a] != ep) {
            stamp[a] = ep;
            st.push_back(a);
        }
        if (stamp[b] != ep) {
            stamp[b] = ep;
            st.push_back(b);
        }
    }
}

// a2: structural support of {var(la), var(lb)} as sorted PI ids; returns AND-cone size.
uint64_t support_of(cec_ctx *c, uint32_t la, uint32_t lb, std::vector<uint32_t> &S) {
    S.clear();
    uint64_t nodes = 0;
    uint32_t roots[2] = {la >> 1, lb >> 1};
    walk_tfi(c, c->scratch, roots, 2, nullptr, 0, [&](uint32_t v) {
        if (v >= 1 && v <= c->I)
            S.push_back(v);
        else if (v > c->I)
            ++nodes;
    });
    std::sort(S.begin(), S.end());
    return nodes;
}

// Schedule builder: topological op order (ascending id, "topological order"), compare
// ops right after their later root, and linear-scan slot allocation by liveness.
struct Sched {
    std::vector<uint4> ops;
    uint32_t nslots = 0;
    uint32_t const_slot = 0xFFFFFFFFu;
};

// Peak number of simultaneously live values of the schedule build_schedule would produce for this
// node order (= its slot count), computed without allocating slots or encoding ops.
uint32_t live_peak(const cec_ctx *c, Scratch &X, const std::vector<uint32_t> &inputs, const std::vector<uint32_t> &nodes,
                   const std::vector<Cmp> &cmps, const std::vector<uint32_t> &win_cmps) {
    X.init(c->N());
    if (++X.sc_epoch == 0) {
        std::fill(X.sc_stamp.begin(), X.sc_stamp.end(), 0u);
        X.sc_epoch = 1;
    }
    const uint32_t ep = X.sc_epoch;
    auto &stamp = X.sc_stamp;
    auto &pos = X.sc_pos;    // 0 = input/const, t+1 = AND node t
    auto &last = X.sc_last;  // last reader position (op index + 1), 0 = never read
    const uint32_t n = (uint32_t)nodes.size(), k = (uint32_t)inputs.size();
    auto touch = [&](uint32_t id) {
        if (stamp[id] != ep) {
            stamp[id] = ep;
            pos[id] = 0;
            last[id] = 0;
        }
    };
    touch(0);
    for (uint32_t id : inputs) touch(id);
    for (uint32_t t = 0; t < n; ++t) {
        touch(nodes[t]);
        pos[nodes[t]] = t + 1;
    }
    // a compare reads its roots right after the later one (op position = that node's position)
    std::vector<uint32_t> cmp_last_reads;  // reader positions of compares, in node-position units
    bool uses_const = false;
    for (uint32_t t = 0; t < n; ++t) {
        const uint32_t id = nodes[t];
        for (uint32_t f : {c->f0[id] >> 1, c->f1[id] >> 1}) {
            touch(f);
            last[f] = std::max(last[f], 2 * (t + 1));  // node t reads at 2(t+1)
            uses_const |= f == 0;
        }
    }
    for (uint32_t ci : win_cmps) {
        const Cmp &cm = cmps[ci];
        touch(cm.la >> 1);
        touch(cm.lb >> 1);
        const uint32_t at = 2 * std::max(pos[cm.la >> 1], pos[cm.lb >> 1]) + 1;  // right after the later root
        last[cm.la >> 1] = std::max(last[cm.la >> 1], at);
        last[cm.lb >> 1] = std::max(last[cm.lb >> 1], at);
        uses_const |= (cm.la >> 1) == 0 || (cm.lb >> 1) == 0;
    }
    // sweep: values die at their last read; an output is born at its node
    std::vector<uint32_t> deaths(2 * n + 3, 0);
    uint32_t live = 0;
    bool const_is_input = false;
    for (uint32_t id : inputs) {
        const_is_input |= id == 0;
        if (last[id]) {
            ++live;
            ++deaths[last[id]];
        }
    }
    uint32_t slots = k + ((uses_const && !const_is_input) ? 1 : 0);  // inputs occupy slots 0..k-1 at pass start
    if (uses_const && !const_is_input) ++live, ++deaths[last[0]];
    uint32_t peak = live;
    for (uint32_t t = 0; t < n; ++t) {
        const uint32_t rd = 2 * (t + 1);
        live -= deaths[rd];  // operands whose last reader is node t are freed before its output
        deaths[rd] = 0;
        ++live;              // node t's output
        if (last[nodes[t]]) ++deaths[last[nodes[t]]];
        else --live;         // never read (cannot happen in a window)
        peak = std::max(peak, live);
        live -= deaths[rd + 1];  // compares placed after node t
        deaths[rd + 1] = 0;
    }
    return std::max(std::max(peak, slots), 1u);
}

bool build_schedule(const cec_ctx *c, Scratch &X, const std::vector<uint32_t> &inputs,
                    const std::vector<uint32_t> &nodes, const std::vector<Cmp> &cmps,
                    const std::vector<uint32_t> &win_cmps, Sched &out, std::string &why) {
    const uint32_t k = (uint32_t)inputs.size();
    const uint32_t n = (uint32_t)nodes.size();
    // per-node scratch, valid where sc_stamp == ep (flat arrays: no hashing on the hot host path)
    X.init(c->N());
    if (++X.sc_epoch == 0) {
        std::fill(X.sc_stamp.begin(), X.sc_stamp.end(), 0u);
        X.sc_epoch = 1;
    }
    const uint32_t ep = X.sc_epoch;
    auto &stamp = X.sc_stamp;
    auto &pos = X.sc_pos;    // 0 = input/const, t+1 = AND node t
    auto &last = X.sc_last;  // last reading op + 1 (0 = never read)
    auto &slot = X.sc_slot;
    auto touch = [&](uint32_t id) {
        if (stamp[id] != ep) {
            stamp[id] = ep;
            pos[id] = 0;
            last[id] = 0;
            slot[id] = 0xFFFFFFFFu;
        }
    };
    touch(0);
    for (uint32_t j = 0; j < k; ++j) touch(inputs[j]);
    for (uint32_t t = 0; t < n; ++t) {
        touch(nodes[t]);
        pos[nodes[t]] = t + 1;
    }
    // compare placement: right after the later root (PAPER.md:118 compares per round; here per pass)
    std::vector<uint32_t> cnt(n + 2, 0);
    std::vector<uint32_t> cmp_at(win_cmps.size());
    for (size_t i = 0; i < win_cmps.size(); ++i) {
        const Cmp &cm = cmps[win_cmps[i]];
        touch(cm.la >> 1);
        touch(cm.lb >> 1);
        cmp_at[i] = std::max(pos[cm.la >> 1], pos[cm.lb >> 1]);  // 0 = before any node
        ++cnt[cmp_at[i] + 1];
    }
    for (uint32_t t = 1; t < n + 2; ++t) cnt[t] += cnt[t - 1];
    std::vector<uint32_t> cmp_sorted(win_cmps.size());
    {
        std::vector<uint32_t> fill(cnt.begin(), cnt.end());
        for (size_t i = 0; i < win_cmps.size(); ++i) cmp_sorted[fill[cmp_at[i]]++] = win_cmps[i];
    }
    // op order: cmps at 0, then node t followed by cmps at t+1
    struct Op { uint32_t la, lb, id; bool cmp; };
    std::vector<Op> order;
    order.reserve(n + win_cmps.size());
    auto push_cmps = [&](uint32_t at) {
        for (uint32_t i = cnt[at]; i < cnt[at + 1]; ++i) {
            const Cmp &cm = cmps[cmp_sorted[i]];
            order.push_back(Op{cm.la, cm.lb, cmp_sorted[i], true});
        }
    };
    push_cmps(0);
    for (uint32_t t = 0; t < n; ++t) {
        const uint32_t id = nodes[t];
        order.push_back(Op{c->f0[id], c->f1[id], id, false});
        push_cmps(t + 1);
    }
    bool uses_const = false;
    for (uint32_t o = 0; o < order.size(); ++o) {
        const uint32_t a = order[o].la >> 1, b = order[o].lb >> 1;
        if (stamp[a] != ep || stamp[b] != ep) {
            why = "schedule: operand outside the window";
            return false;
        }
        last[a] = o + 1;
        last[b] = o + 1;
        uses_const |= (a == 0 || b == 0);
    }
    std::vector<uint32_t> free_list;
    uint32_t next = k;
    for (uint32_t j = 0; j < k; ++j) slot[inputs[j]] = j;
    bool const_is_input = false;
    for (uint32_t j = 0; j < k; ++j) const_is_input |= inputs[j] == 0;
    if (uses_const && !const_is_input) {
        out.const_slot = next++;
        slot[0] = out.const_slot;
    }
    for (uint32_t j = k; j-- > 0;)  // inputs never read are free from the start
        if (!last[inputs[j]]) free_list.push_back(j);
    out.ops.clear();
    out.ops.reserve(order.size());
    for (uint32_t o = 0; o < order.size(); ++o) {
        const Op &op = order[o];
        const uint32_t va = op.la >> 1, vb = op.lb >> 1;
        if (slot[va] == 0xFFFFFFFFu || slot[vb] == 0xFFFFFFFFu) {
            why = "schedule: operand not defined before use";
            return false;
        }
        uint4 e;
        e.x = slot[va] * SLOT_BYTES | (op.la & 1u);
        e.y = slot[vb] * SLOT_BYTES | (op.lb & 1u);
        e.w = 0;
        // free operands whose last reader is this op (the kernel reads before it writes)
        if (last[va] == o + 1) free_list.push_back(slot[va]);
        if (vb != va && last[vb] == o + 1) free_list.push_back(slot[vb]);
        if (op.cmp) {
            e.z = OP_CMP | op.id;
        } else {
            uint32_t s;
            if (!free_list.empty()) {
                s = free_list.back();
                free_list.pop_back();
            } else {
                s = next++;
            }
            if (s >= MAX_SLOTS) {
                why = "schedule: live set exceeds the slot field";
                return false;
            }
            slot[op.id] = s;
            e.z = s * SLOT_BYTES;
            if (!last[op.id]) free_list.push_back(s);  // never read (cannot happen in a window)
        }
        out.ops.push_back(e);
    }
    out.nslots = std::max<uint32_t>(next, 1);
    return true;
}

}  // namespace

// ------------------------------------------------------------------------------------------------
// ABI
// ------------------------------------------------------------------------------------------------
extern "C" {

int cec_abi_version(void) { return CEC_ABI_VERSION; }

void cec_default_opts(cec_opts *o) {
    if (!o) return;
    std::memset(o, 0, sizeof *o);
    o->device = 0;
    o->rank = 0;
    o->world = 1;
    o->k_max = 32;
    o->k_s = 0;
    o->merge = CEC_MERGE_PAPER;
    o->engine = CEC_ENGINE_AUTO;
}

const char *cec_last_error(const cec_ctx *ctx) { return ctx ? ctx->err.c_str() : g_load_err.c_str(); }

void cec_shard_range(uint64_t n, int32_t rank, int32_t world, uint64_t *begin, uint64_t *end) {
    if (world < 1) world = 1;
    unsigned __int128 b = (unsigned __int128)n * (uint64_t)rank / (uint64_t)world;
    unsigned __int128 e = (unsigned __int128)n * (uint64_t)(rank + 1) / (uint64_t)world;
    *begin = (uint64_t)b;
    *end = (uint64_t)e;
}

cec_status cec_nccl_unique_id(void *out128) {
    if (!out128) return CEC_E_ARG;
    if (!g_nccl.load()) return fail(nullptr, CEC_E_NCCL, "NCCL library not found");
    ncclUniqueId id;
    ncclResult_t r = g_nccl.get_id(&id);
    if (r != ncclSuccess) return fail(nullptr, CEC_E_NCCL, "ncclGetUniqueId: %s", g_nccl.err(r));
    std::memcpy(out128, &id, sizeof id);
    return CEC_OK;
}

cec_status cec_peer_export(cec_ctx *c, void *blob_out) {
    if (!c || !blob_out) return CEC_E_ARG;
    if (c->host_only) return fail(c, CEC_E_CUDA, "host-only context: no CUDA device");
    if (c->opts.world < 2 || c->opts.world > PEER_MAX) return fail(c, CEC_E_ARG, "peer mode needs 2 <= world <= 8");
    const char *e = peer_export(c->peer, c->opts.device, c->opts.rank, c->opts.world, blob_out);
    return e ? fail(c, CEC_E_CUDA, "CUDA: %s (peer export)", e) : CEC_OK;
}

cec_status cec_peer_import(cec_ctx *c, const void *blobs) {
    if (!c || !blobs) return CEC_E_ARG;
    if (c->host_only) return fail(c, CEC_E_CUDA, "host-only context: no CUDA device");
    const char *e = peer_import(c->peer, c->opts.device, c->opts.rank, c->opts.world, blobs);
    return e ? fail(c, CEC_E_CUDA, "peer import: %s", e) : CEC_OK;
}

cec_status cec_peer_host_barrier(cec_ctx *c, void (*fn)(void *), void *user) {
    if (!c) return CEC_E_ARG;
    if (!c->peer.on) return fail(c, CEC_E_STATE, "cec_peer_host_barrier needs a connected peer context");
    c->peer.host_barrier = fn;
    c->peer.host_user = user;
    ++c->peer.gen;  // graphs captured with device barriers are stale
    return CEC_OK;
}

uint64_t cec_pext64(uint64_t value, uint64_t mask) {
    uint64_t r = 0;
    int j = 0;
    for (int b = 0; b < 64; ++b) {
        if ((mask >> b) & 1u) {
            r |= ((value >> b) & 1u) << j;
            ++j;
        }
    }
    return r;
}

}  // extern "C"

// a1: validate the AIGER arrays (fanin id < own id, PO literals in range) and
// compute levels into temporaries; only a valid AIG replaces the context's arrays.
static cec_status set_aig(cec_ctx *c, const cec_aig *aig, std::string &err) {
    if (aig->num_ands && !aig->fanin_lits) return CEC_E_ARG;
    const uint64_t N = 1ull + aig->num_pis + aig->num_ands;
    if (N >= (1ull << 31)) return CEC_E_ARG;
    const uint32_t I = aig->num_pis, A = aig->num_ands, O = aig->num_pos;
    std::vector<uint32_t> f0, f1, level;
    try {
        f0.assign(N, 0);
        f1.assign(N, 0);
        level.assign(N, 0);
    } catch (...) {
        return CEC_E_NOMEM;
    }
    for (uint32_t i = 0; i < A; ++i) {
        const uint32_t id = 1 + I + i;
        const uint32_t l0 = aig->fanin_lits[2 * i], l1 = aig->fanin_lits[2 * i + 1];
        if ((l0 >> 1) >= id || (l1 >> 1) >= id) {
            err = "AIG: fanin id >= own id at AND " + std::to_string(id);
            return CEC_E_AIG;
        }
        f0[id] = l0;
        f1[id] = l1;
        level[id] = 1 + std::max(level[l0 >> 1], level[l1 >> 1]);
    }
    for (uint32_t i = 0; i < O; ++i)
        if (aig->po_lits && (aig->po_lits[i] >> 1) >= N) {
            err = "AIG: PO literal out of range";
            return CEC_E_AIG;
        }
    c->I = I;
    c->A = A;
    c->O = O;
    c->f0.swap(f0);
    c->f1.swap(f1);
    c->level.swap(level);
    return CEC_OK;
}

extern "C" {

cec_status cec_load_aig(cec_ctx **out, const cec_aig *aig, const cec_opts *opts) {
    if (!out || !aig) return CEC_E_ARG;
    *out = nullptr;
    std::unique_ptr<cec_ctx> c(new (std::nothrow) cec_ctx());
    if (!c) return CEC_E_NOMEM;
    cec_default_opts(&c->opts);
    if (opts) c->opts = *opts;
    if (c->opts.k_max > 63) return fail(nullptr, CEC_E_ARG, "k_max > 63");
    if (c->opts.k_s == 0) c->opts.k_s = c->opts.k_max;
    if (c->opts.world < 1) c->opts.world = 1;
    if (c->opts.rank < 0 || c->opts.rank >= c->opts.world) return CEC_E_ARG;
    std::string err;
    const cec_status st = set_aig(c.get(), aig, err);  // a1: validation and levels
    if (st != CEC_OK) return err.empty() ? st : fail(nullptr, st, "%s", err.c_str());
    if (c->opts.device >= 0) {
        c->host_only = false;
        const char *e = dev_init(c->opts.device, &c->own_stream, &c->num_sms);
        if (e) {
            // keep the context only to report the error through the status
            return CEC_E_CUDA;
        }
        c->stream = c->opts.stream ? c->opts.stream : c->own_stream;
        if (getenv("CEC_NO_SIDE_STREAMS") == nullptr) {
            const char *ea = aux_create(c->aux);
            if (ea) return fail(nullptr, CEC_E_CUDA, "CUDA: %s (side streams)", ea);
        }
        if (c->opts.nccl_unique_id) {  // NULL id with world > 1: shard-only mode, no collective
            if (!g_nccl.load()) return fail(nullptr, CEC_E_NCCL, "NCCL library not found");
            ncclUniqueId uid;
            std::memcpy(&uid, c->opts.nccl_unique_id, sizeof uid);
            ncclResult_t r = g_nccl.init_rank(&c->comm, c->opts.world, uid, c->opts.rank);
            if (r != ncclSuccess) return CEC_E_NCCL;
        }
    }
    *out = c.release();
    return CEC_OK;
}

void cec_free(cec_ctx *ctx) {
    if (!ctx) return;
    dev_free(ctx->d_f0);
    dev_free(ctx->d_f1);
    dev_free(ctx->d_level_ids);
    dev_free(ctx->supp_table.lists);
    if (ctx->comm && g_nccl.destroy) g_nccl.destroy(ctx->comm);
    if (ctx->peer.own) {
        stream_sync(ctx->stream);
        peer_close(ctx->peer);
    }
    aux_destroy(ctx->aux);
    ctx->devpool.reset();  // freed here unless a live plan still holds it
    if (ctx->own_stream) stream_destroy(ctx->own_stream);
    delete ctx;
}

cec_status cec_reload_aig(cec_ctx *c, const cec_aig *aig, uint32_t k_max, uint32_t k_s) {
    if (!c || !aig) return CEC_E_ARG;
    if (k_max > 63) return fail(c, CEC_E_ARG, "k_max > 63");
    if (!c->host_only) {  // nothing of the old AIG may still be in flight
        const char *e = stream_sync(c->stream);
        if (e) return fail(c, CEC_E_CUDA, "CUDA: %s (reload)", e);
    }
    std::string err;
    const cec_status st = set_aig(c, aig, err);
    if (st != CEC_OK) return fail(c, st, "%s", err.empty() ? "invalid AIG arrays" : err.c_str());
    // everything derived from the old AIG: its device copy + level CSR, the per-node support table,
    // the last global check (cec_get_cex)
    // the device AIG buffers are kept for the next upload (a reduced miter fits: cudaFree /
    // cudaMalloc here cost up to 0.5 s spikes per phase on the B200 box); only their data is stale
    c->d_aig_valid = false;
    dev_free(c->supp_table.lists);
    c->supp_table = NodeSupports{};
    c->level_off.clear();
    c->have_last = false;
    c->last_verdict.clear();
    c->last_cex.clear();
    c->last_support.clear();
    if (k_max) {
        c->opts.k_max = k_max;
        c->opts.k_s = k_s ? k_s : k_max;
    } else if (k_s) {
        c->opts.k_s = k_s;
    }
    return CEC_OK;
}

void *cec_stream(cec_ctx *ctx) { return ctx ? ctx->stream : nullptr; }

cec_status cec_get_stats(cec_ctx *ctx, cec_stats *s) {
    if (!ctx || !s) return CEC_E_ARG;
    *s = ctx->stats;
    return CEC_OK;
}

cec_status cec_pair_support(cec_ctx *ctx, uint32_t la, uint32_t lb, uint32_t *sup, uint32_t cap, uint32_t *k_out) {
    if (!ctx || !k_out) return CEC_E_ARG;
    if ((la >> 1) >= ctx->N() || (lb >> 1) >= ctx->N()) return fail(ctx, CEC_E_ARG, "literal out of range");
    std::vector<uint32_t> S;
    support_of(ctx, la, lb, S);
    for (uint32_t j = 0; j < cap && j < S.size(); ++j) sup[j] = S[j];
    *k_out = (uint32_t)S.size();
    return CEC_OK;
}

}  // extern "C"

// ------------------------------------------------------------------------------------------------
// Planning
// ------------------------------------------------------------------------------------------------
namespace {

constexpr int32_t DECIDED_BY_SIM = -100;
// Slice indices are 32-bit (2^(k-10) JIT slices): windows above 2^41 patterns are never enumerated
// (they would take days even at the LOP3 peak); such pairs are UNDECIDED like k > k_max.
constexpr size_t MAX_K_ENUM = 41;
JitConfig jit_config() {  // overridable for tuning: CEC_JIT_THREADS / CEC_JIT_MINB / CEC_JIT_SYNC
    JitConfig cfg;
    if (const char *e = getenv("CEC_JIT_THREADS")) cfg.threads = atoi(e);
    if (const char *e = getenv("CEC_JIT_MINB")) cfg.min_blocks = atoi(e);
    if (const char *e = getenv("CEC_JIT_SYNC")) cfg.sync_every = atoi(e);
    if (const char *e = getenv("CEC_JIT_FUSE")) cfg.fuse = atoi(e);
    if (const char *e = getenv("CEC_JIT_SPLICE")) cfg.splice = atoi(e) != 0;
    return cfg;
}

uint64_t tt_words_of(uint32_t k) { return k <= 5 ? 1ull : (1ull << (k - 5)); }

// Build per-window programs, work items and launch groups; compute W. Common to global and local.
struct PhaseTimer {  // CEC_TIMING=1: per-phase host timings on stderr
    bool on = getenv("CEC_TIMING") != nullptr;
    std::chrono::steady_clock::time_point t = std::chrono::steady_clock::now();
    void lap(const char *what) {
        if (!on) return;
        auto n = std::chrono::steady_clock::now();
        fprintf(stderr, "[cec] %-28s %8.2f ms\n", what, std::chrono::duration<double, std::milli>(n - t).count());
        t = n;
    }
};

cec_status finish_plan(cec_ctx *c, cec_plan *P, std::vector<WinHost> &wins, const std::vector<uint32_t> *stop,
                       bool local) {
    PhaseTimer tm;
    const int32_t rank = c->opts.rank, world = c->opts.world;
    P->dwin.clear();
    P->prog.clear();
    P->items.clear();
    P->jitems.clear();
    P->joff.clear();
    P->groups.clear();
    P->win_inputs.clear();
    P->win_nodes.clear();
    P->win_cmps.clear();
    // Re-number compares window by window so each window's compares are contiguous.
    std::vector<Cmp> cmps2;
    cmps2.reserve(P->cmps.size());
    std::vector<int32_t> remap(P->cmps.size(), -1);
    const uint32_t max_slot_cap = interp_max_slots_per_warp();
    std::vector<uint32_t> nslots_of;
    std::vector<uint64_t> cost_of;
    std::vector<int32_t> win_jit;                    // JIT structure index per window, -1 = interpreter
    std::vector<uint64_t> wps_of;                    // words per slice per window
    std::vector<uint64_t> words_rank_of;             // u32 words this rank simulates per window
    std::vector<JitProgram> jit_progs;
    std::unordered_map<uint64_t, uint32_t> jit_hindex;  // structure hash -> program index
    std::vector<uint32_t> jit_rep;                      // program index -> window it was taken from
    // (1) serial: lay out compares window by window (contiguous per window) and own-support masks
    std::vector<std::vector<uint32_t>> wcs(wins.size());
    for (size_t w = 0; w < wins.size(); ++w) {
        for (uint32_t ci : wins[w].cmps) {
            remap[ci] = (int32_t)cmps2.size();
            wcs[w].push_back((uint32_t)cmps2.size());
            cmps2.push_back(std::move(P->cmps[ci]));  // each compare sits in one window
        }
        for (uint32_t ci : wcs[w]) {  // a11 pext masks
            Cmp &cm = cmps2[ci];
            uint64_t m = 0;
            size_t j = 0;
            for (size_t t = 0; t < wins[w].inputs.size() && j < cm.S.size(); ++t) {
                if (wins[w].inputs[t] == cm.S[j]) {
                    m |= 1ull << t;
                    ++j;
                }
            }
            cm.ownmask = m;
        }
    }
    // AUTO engine: a window is compiled when its sweep is at least this many node-words
    uint64_t jit_min_node_words = 1ull << 20;
    if (const char *e = getenv("CEC_JIT_MIN_NODE_WORDS")) jit_min_node_words = strtoull(e, nullptr, 10);
    // (2) parallel over windows: node order, schedule, engine choice, JIT program
    struct WinRes {
        std::vector<uint32_t> nodes;
        Sched sc;
        bool jit = false;
        JitProgram jp;
        std::string key, err;
        uint64_t hkey = 0;  // 64-bit hash of key (computed in parallel; exact compare verifies)
    };
    std::vector<WinRes> res(wins.size());
    auto plan_one = [&](size_t w, Scratch &X) {
        WinHost &W = wins[w];
        WinRes &R = res[w];
        const std::vector<uint32_t> &wc = wcs[w];
        std::vector<uint32_t> roots;
        for (uint32_t ci : wc) {
            roots.push_back(cmps2[ci].la >> 1);
            roots.push_back(cmps2[ci].lb >> 1);
        }
        X.init(c->N());
        const uint32_t sep = X.next_stop();  // window inputs stop the backward traversal (Q6)
        for (uint32_t x : W.inputs) X.stop[x] = sep;
        // Node order = a topological order chosen to keep the live set small (it sets the
        // interpreter's shared-memory slots and the JIT kernel's register pressure): depth-first
        // post-order from the roots, compare by compare, deeper fanin first (Sethi-Ullman style).
        std::vector<uint32_t> &nodes = R.nodes;
        {
            const uint32_t ep = X.next_epoch();
            // raw pointers: the loop is latency-bound on these lookups (no vector reloads)
            const uint32_t *f0 = c->f0.data(), *f1 = c->f1.data(), *lvl = c->level.data();
            uint32_t *stamp = X.stamp.data();
            const uint32_t *stop = X.stop.data();
            const uint32_t I = c->I;
            std::vector<uint32_t> st;  // node << 1 | (second fanin done)
            st.reserve(256);
            nodes.reserve(1024);
            auto enter = [&](uint32_t x) { return stamp[x] != ep && x > I && stop[x] != sep; };
            for (uint32_t r : roots) {
                if (!enter(r)) continue;
                stamp[r] = ep;
                st.push_back(r << 1);
                while (!st.empty()) {
                    const uint32_t top = st.back(), v = top >> 1;
                    uint32_t a = f0[v] >> 1, b = f1[v] >> 1;
                    if (lvl[b] > lvl[a]) std::swap(a, b);  // deeper fanin first
                    if (!(top & 1u)) {  // first visit: descend into a (then b)
                        st.back() = top | 1u;
                        if (enter(a)) {
                            stamp[a] = ep;
                            st.push_back(a << 1);
                            continue;
                        }
                    }
                    // a done: descend into b unless done, else emit v
                    if (enter(b)) {
                        stamp[b] = ep;
                        st.push_back(b << 1);
                        continue;
                    }
                    nodes.push_back(v);
                    st.pop_back();
                }
            }
        }
        // the id order (the netlist's own construction order) is often the better one: keep the
        // order with the smaller live set (counted without building the schedule)
        std::string why;
        // An interpreter window whose depth-first order already fits the smallest slot bucket (32
        // slots: the launch configuration cannot get better) skips the id-order evaluation.
        const uint32_t kw = (uint32_t)W.inputs.size();
        const uint64_t nw_est = (uint64_t)nodes.size() * tt_words_of(kw);
        const bool interp_bound =
            c->opts.engine == CEC_ENGINE_INTERP ||
            (c->opts.engine == CEC_ENGINE_AUTO &&
             (kw < 10 || nw_est < (kw <= 16 ? jit_min_node_words << 3 : jit_min_node_words)));
        const uint32_t l_dfs0 = interp_bound ? live_peak(c, X, W.inputs, nodes, cmps2, wc) : UINT32_MAX;
        if (interp_bound && l_dfs0 <= 32) {
            R.sc.nslots = l_dfs0;
        } else {
            // ascending ids: a flag scan over the window's id range (ids of a window are dense
            // in practice: one copy / one block), else a sort
            std::vector<uint32_t> by_id;
            by_id.reserve(nodes.size());
            uint32_t lo = UINT32_MAX, hi = 0;
            for (uint32_t v : nodes) lo = std::min(lo, v), hi = std::max(hi, v);
            if (!nodes.empty() && (uint64_t)(hi - lo) + 1 <= 8 * (uint64_t)nodes.size() + 64) {
                std::vector<uint8_t> flag(hi - lo + 1, 0);
                for (uint32_t v : nodes) flag[v - lo] = 1;
                for (uint32_t i = 0; i <= hi - lo; ++i)
                    if (flag[i]) by_id.push_back(lo + i);
            } else {  // two or more clusters (e.g. a block of A and its image in B): LSD radix sort
                by_id = nodes;
                std::vector<uint32_t> tmp(by_id.size());
                for (int sh = 0; sh < 32 && (hi >> sh) != 0; sh += 11) {
                    uint32_t cnt[2049] = {0};
                    for (uint32_t v : by_id) ++cnt[((v >> sh) & 2047u) + 1];
                    for (int b = 0; b < 2048; ++b) cnt[b + 1] += cnt[b];
                    for (uint32_t v : by_id) tmp[cnt[(v >> sh) & 2047u]++] = v;
                    by_id.swap(tmp);
                }
            }
            const uint32_t l_id = live_peak(c, X, W.inputs, by_id, cmps2, wc);
            const uint32_t l_dfs = l_dfs0 != UINT32_MAX ? l_dfs0 : live_peak(c, X, W.inputs, nodes, cmps2, wc);
            if (l_id < l_dfs) nodes.swap(by_id);
            R.sc.nslots = std::min(l_id, l_dfs);
        }
        const uint32_t k = (uint32_t)W.inputs.size();
        // engine choice: straight-line register kernel for big windows (k >= 10 so a 32-word warp
        // pass is never partial); the interpreter for small ones (JIT compile would dominate)
        const uint64_t node_words = (uint64_t)nodes.size() * tt_words_of(k);
        if (k >= 10 && !nodes.empty()) {
            if (c->opts.engine == CEC_ENGINE_JIT) R.jit = true;
            else if (c->opts.engine == CEC_ENGINE_SIMT && !local) R.jit = false;
            else if (c->opts.engine == CEC_ENGINE_AUTO)
                // k <= 16 windows (local checks, G-phase pairs, the sweeping flow's re-planned
                // miters) finish in microseconds on the interpreter: compiling them pays only in
                // repeated runs of one plan, so they need 8x the work of larger-k windows
                R.jit = node_words >= (k <= 16 ? jit_min_node_words << 3 : jit_min_node_words) ||
                        R.sc.nslots > max_slot_cap;
        }
        if (!R.jit && !(c->opts.engine == CEC_ENGINE_SIMT && !local)) {  // interpreter program
            if (!build_schedule(c, X, W.inputs, nodes, cmps2, wc, R.sc, why)) {
                R.err = why;
                return;
            }
        }
        if (!R.jit && R.sc.nslots > max_slot_cap && !(c->opts.engine == CEC_ENGINE_SIMT && !local)) {
            char b[160];
            snprintf(b, sizeof b, "window %zu needs %u live slots > %u (shared-memory capacity)", w, R.sc.nslots,
                     max_slot_cap);
            R.err = b;
            return;
        }
        if (R.jit) {  // SSA program: refs via the per-thread flat arrays (inputs 1..k, nodes k+1..)
            JitProgram &jp = R.jp;
            jp.k = k;
            if (++X.sc_epoch == 0) {
                std::fill(X.sc_stamp.begin(), X.sc_stamp.end(), 0u);
                X.sc_epoch = 1;
            }
            const uint32_t ep = X.sc_epoch;
            auto setref = [&](uint32_t id, uint32_t r) {
                X.sc_stamp[id] = ep;
                X.sc_pos[id] = r;
            };
            auto ref = [&](uint32_t id) { return id == 0 ? 0u : X.sc_pos[id]; };
            for (uint32_t j = 0; j < k; ++j) setref(W.inputs[j], j + 1);
            for (uint32_t t = 0; t < nodes.size(); ++t) setref(nodes[t], k + 1 + t);
            jp.nodes.reserve(2 * nodes.size());
            for (uint32_t id : nodes) {
                jp.nodes.push_back(ref(c->f0[id] >> 1) << 1 | (c->f0[id] & 1u));
                jp.nodes.push_back(ref(c->f1[id] >> 1) << 1 | (c->f1[id] & 1u));
            }
            for (uint32_t ci : wc) {
                jp.cmps.push_back(ref(cmps2[ci].la >> 1) << 1 | (cmps2[ci].la & 1u));
                jp.cmps.push_back(ref(cmps2[ci].lb >> 1) << 1 | (cmps2[ci].lb & 1u));
            }
            R.key = jit_key(jp);
            uint64_t h = 0x9E3779B97F4A7C15ull ^ R.key.size();  // word-wise multiply-xorshift hash
            const uint64_t *q = reinterpret_cast<const uint64_t *>(R.key.data());
            const size_t nq = R.key.size() / 8;
            for (size_t i = 0; i < nq; ++i) {
                uint64_t v = q[i] * 0xBF58476D1CE4E5B9ull;
                h = (h ^ (v ^ (v >> 31))) * 0x94D049BB133111EBull;
            }
            for (size_t i = nq * 8; i < R.key.size(); ++i) h = (h ^ (uint8_t)R.key[i]) * 0x100000001B3ull;
            R.hkey = h ^ (h >> 29);
        }
    };
    if (wins.size() < 2) {
        for (size_t w = 0; w < wins.size(); ++w) plan_one(w, c->scratch);
    } else {  // persistent per-thread scratch (no per-call allocation), persistent workers
        WorkPool &wp = c->workers();
        wp.run((uint32_t)wins.size(), [&](uint32_t w, unsigned tid) { plan_one(w, c->pool[tid]); });
    }
    tm.lap("per-window plans (parallel)");
    size_t prog_total = 0;
    // Multi-GPU split: a window with at least `world` slices is cut into
    // contiguous slice ranges, one per rank; a smaller window goes WHOLE to one rank, chosen by
    // longest-processing-time-first over the node-words of the small windows on top of each rank's
    // share of the big ones (deterministic: every rank plans the same assignment). The min-reduce
    // of the results is unchanged: a rank that does not simulate a window reports no mismatch.
    std::vector<int32_t> owner(wins.size(), -1);
    if (world > 1) {
        std::vector<uint64_t> load(world, 0);
        std::vector<std::pair<uint64_t, uint32_t>> small;
        for (uint32_t w = 0; w < wins.size(); ++w) {
            const uint32_t k = (uint32_t)wins[w].inputs.size();
            const uint64_t ttw = tt_words_of(k), wps = res[w].jit ? 32 : 32 * IV;
            const uint64_t slices = (ttw + wps - 1) / wps, cost = (uint64_t)res[w].nodes.size() * ttw + 1;
            if (slices >= (uint64_t)world) {
                for (int32_t r = 0; r < world; ++r) load[r] += cost / world;
            } else {
                small.push_back({cost, w});
            }
        }
        std::stable_sort(small.begin(), small.end(),
                         [](const std::pair<uint64_t, uint32_t> &a, const std::pair<uint64_t, uint32_t> &b) {
                             return a.first > b.first;
                         });
        for (const auto &sw : small) {
            int32_t best = 0;
            for (int32_t r = 1; r < world; ++r)
                if (load[r] < load[best]) best = r;
            owner[sw.second] = best;
            load[best] += sw.first;
        }
    }
    auto win_range = [&](uint32_t w, uint64_t slices, uint64_t *sb, uint64_t *se) {
        if (owner[w] < 0) {
            cec_shard_range(slices, rank, world, sb, se);
        } else {
            *sb = 0;
            *se = owner[w] == rank ? slices : 0;
        }
    };
    // (3) serial assembly in window order
    for (size_t w = 0; w < wins.size(); ++w) {
        WinHost &W = wins[w];
        WinRes &R = res[w];
        if (!R.err.empty()) return fail(c, CEC_E_NOMEM, "%s", R.err.c_str());
        const std::vector<uint32_t> &wc = wcs[w];
        const std::vector<uint32_t> &nodes = R.nodes;
        const Sched &sc = R.sc;
        DevWin dw{};
        dw.cmp_off = wc.empty() ? (uint32_t)cmps2.size() : wc[0];
        dw.ncmp = (uint32_t)wc.size();
        dw.prog_off = (uint32_t)prog_total;
        dw.prog_len = R.jit ? 0u : (uint32_t)sc.ops.size();  // JIT windows need no interpreter ops
        prog_total += dw.prog_len;
        dw.k = (uint32_t)W.inputs.size();
        dw.const_slot = sc.const_slot;
        const uint64_t ttw = tt_words_of(dw.k);
        dw.tt_words_lo = (uint32_t)ttw;
        dw.tt_words_hi = (uint32_t)(ttw >> 32);
        P->dwin.push_back(dw);
        P->win_nodes.push_back((uint32_t)nodes.size());
        if (c->opts.engine == CEC_ENGINE_SIMT && !local) {  // the Alg. 1 layout below reads them again
            P->win_inputs.push_back(W.inputs);
            P->win_cmps.push_back(wc);
        } else {  // the caller's windows are discarded after planning: no copies
            P->win_inputs.push_back(std::move(W.inputs));
            P->win_cmps.push_back(std::move(wcs[w]));
        }
        nslots_of.push_back(sc.nslots);
        const bool jit = R.jit;
        if (jit) {  // windows of identical structure share one program (by hash; verified below)
            auto it = jit_hindex.find(R.hkey);
            if (it == jit_hindex.end()) {
                it = jit_hindex.emplace(R.hkey, (uint32_t)jit_progs.size()).first;
                R.jp.key = R.key;  // the cache lookup's key part (R.key stays for the exact verify)
                jit_progs.push_back(std::move(R.jp));
                jit_rep.push_back((uint32_t)w);
            }
            win_jit.push_back((int32_t)it->second);
        } else {
            win_jit.push_back(-1);
        }
        P->max_k = std::max(P->max_k, dw.k);
        P->max_slots = std::max(P->max_slots, sc.nslots);
        const uint64_t wps = jit ? 32 : 32 * IV;  // words per slice of this window's engine
        wps_of.push_back(wps);
        // W accounting: nodes x patterns, per rank and all ranks
        const uint64_t slices = (ttw + wps - 1) / wps;
        if (dw.k > MAX_K_ENUM || slices > UINT32_MAX)  // work items carry u32 slice bounds
            return fail(c, CEC_E_ARG, "window %zu: k = %u exceeds the enumeration limit %zu", w, dw.k, MAX_K_ENUM);
        const uint64_t pats_all = dw.k < 5 ? (1ull << dw.k) : ttw * 32;
        P->W_all += (uint64_t)nodes.size() * pats_all;
        uint64_t sb, se;
        win_range((uint32_t)w, slices, &sb, &se);
        uint64_t wb = sb * wps, we = std::min<uint64_t>(se * wps, ttw);
        uint64_t pats_rank = we > wb ? (dw.k < 5 ? (1ull << dw.k) : (we - wb) * 32) : 0;
        P->W_rank += (uint64_t)nodes.size() * pats_rank;
        words_rank_of.push_back(we > wb ? (we - wb) : 0);
        cost_of.push_back((uint64_t)(sc.ops.size() + 1) * (se - sb));
    }
    tm.lap("layout: serial window loop");
    {  // interpreter programs copied into their slots of one array in parallel
        P->prog.resize(prog_total);
        auto copy = [&](uint32_t w, unsigned) {
            if (!res[w].jit && !res[w].sc.ops.empty())
                std::copy(res[w].sc.ops.begin(), res[w].sc.ops.end(), P->prog.begin() + P->dwin[w].prog_off);
        };
        if (wins.size() < 2 || prog_total < (1u << 16)) {  // small: a pool hand-off costs more than the copy
            for (uint32_t w = 0; w < wins.size(); ++w) copy(w, 0);
        } else {
            c->workers().run((uint32_t)wins.size(), copy);
        }
    }
    tm.lap("per-window serial layout");
    {  // exactness of the hash dedupe: every window's structure key equals its program's (parallel
       // memcmp); a 64-bit collision (never seen) gets its own program through an exact-key map
        std::vector<uint8_t> bad(wins.size(), 0);
        auto verify = [&](uint32_t w, unsigned) {
            const int32_t pi = win_jit[w];
            if (pi >= 0 && jit_rep[pi] != w && res[w].key != res[jit_rep[pi]].key) bad[w] = 1;
        };
        size_t njit = 0;  // only JIT windows have keys to compare
        for (uint32_t w = 0; w < wins.size(); ++w) njit += win_jit[w] >= 0;
        if (njit < 64) {
            for (uint32_t w = 0; w < wins.size(); ++w) verify(w, 0);
        } else {
            c->workers().run((uint32_t)wins.size(), verify);
        }
        std::unordered_map<std::string, uint32_t> exact;
        for (uint32_t w = 0; w < wins.size(); ++w) {
            if (!bad[w]) continue;
            auto it = exact.find(res[w].key);
            if (it == exact.end()) {
                it = exact.emplace(res[w].key, (uint32_t)jit_progs.size()).first;
                jit_progs.push_back(std::move(res[w].jp));
                jit_rep.push_back(w);
            }
            win_jit[w] = (int32_t)it->second;
        }
    }
    tm.lap("structure dedupe (hash)");
    if (c->opts.engine == CEC_ENGINE_SIMT && !local) {  // the paper's Alg. 1 layout (sim_simt.cu)
        if (world != 1) return fail(c, CEC_E_ARG, "CEC_ENGINE_SIMT runs on one GPU (world = 1)");
        SimtPlan &S = P->simt;
        S = SimtPlan{};
        std::vector<uint32_t> row_of(c->N(), 0), lvl_of(c->N(), 0);
        uint64_t rows = 1;  // row 0 = constant 0
        std::vector<std::vector<uint4>> by_level;
        uint64_t max_ttw = 1;
        for (size_t w = 0; w < wins.size(); ++w) {
            const WinHost &W = wins[w];
            const uint32_t k = (uint32_t)W.inputs.size();
            max_ttw = std::max<uint64_t>(max_ttw, tt_words_of(k));
            S.h_ttw.push_back(tt_words_of(k));
            row_of[0] = 0;
            lvl_of[0] = 0;
            for (uint32_t j = 0; j < k; ++j) {
                row_of[W.inputs[j]] = (uint32_t)rows;
                lvl_of[W.inputs[j]] = 0;
                S.h_inputs.push_back(make_uint4((uint32_t)rows++, (uint32_t)w, j, 0));
            }
            for (uint32_t id : res[w].nodes) {  // topological: fanins are inputs, 0 or earlier nodes
                const uint32_t a = c->f0[id] >> 1, b = c->f1[id] >> 1;
                const uint32_t l = 1 + std::max(lvl_of[a], lvl_of[b]);  // window level, inputs at 0
                lvl_of[id] = l;
                row_of[id] = (uint32_t)rows++;
                if (by_level.size() <= l) by_level.resize(l + 1);
                by_level[l].push_back(make_uint4(row_of[id], row_of[a] | (c->f0[id] & 1u) << 31,
                                                 row_of[b] | (c->f1[id] & 1u) << 31, (uint32_t)w));
            }
            for (uint32_t ci : wcs[w]) {
                const Cmp &cm = cmps2[ci];
                S.h_pairs.push_back(make_uint4(row_of[cm.la >> 1] | (cm.la & 1u) << 31,
                                               row_of[cm.lb >> 1] | (cm.lb & 1u) << 31, (uint32_t)w, ci));
            }
        }
        for (auto &l : by_level) {
            S.level_off.push_back((uint32_t)S.h_nodes.size());
            S.h_nodes.insert(S.h_nodes.end(), l.begin(), l.end());
        }
        S.level_off.push_back((uint32_t)S.h_nodes.size());
        uint64_t M = 16384ull << 18;  // words (16 GiB)
        if (const char *e = getenv("CEC_SIMT_MB")) M = strtoull(e, nullptr, 10) << 18;
        if (c->opts.workspace) M = c->opts.workspace_bytes / 4;  // the caller's budget (Alg. 1 input M)
        uint64_t E = 4;  // Alg. 1 l.2: the largest power of two with E x rows <= M
        while (E * 2 * rows <= M && E < max_ttw) E *= 2;
        if (E * rows > M) return fail(c, CEC_E_NOMEM, "simulation table: %llu rows do not fit M", (unsigned long long)rows);
        S.E = (uint32_t)E;
        S.rows = rows;
        S.rounds = (max_ttw + E - 1) / E;  // Alg. 1 l.4, with the ceiling (reading Q5)
        S.n_inputs = (uint32_t)S.h_inputs.size();
        S.n_pairs = (uint32_t)S.h_pairs.size();
        P->groups.clear();
        P->items.clear();
        P->jitems.clear();
    }
    tm.lap("windows+schedules+jit-progs");
    P->cmps.swap(cmps2);
    for (auto &pc : P->pair_cmp)
        if (pc >= 0) pc = remap[pc];
    // compile the distinct JIT structures (in parallel; cached process-wide by structure)
    if (P->simt.E) {  // no JIT kernels / work items for Alg. 1 plans
        P->jit_kernels = 0;
        P->jit_windows = 0;
        P->lop3_words = 0;
        for (size_t w = 0; w < wins.size(); ++w) P->lop3_words += (uint64_t)P->win_nodes[w] * words_rank_of[w];
        return CEC_OK;
    }
    const JitConfig jcfg = jit_config();
    const uint64_t jit_pass = jcfg.sync_every > 0 ? (uint64_t)jcfg.threads / 32 : 1;
    // Compile units: a structure whose windows fill the GPU on their own gets its own kernel; the
    // others (typically single small windows) are packed into bundle kernels (jit_source_bundle)
    // so one persistent grid runs all of them instead of many tiny launches.
    std::vector<std::vector<uint32_t>> units;  // program indices per compiled kernel
    std::vector<uint32_t> unit_of(jit_progs.size(), 0), sid_of(jit_progs.size(), 0);
    {
        // a structure runs standalone when its sweep is long next to a launch's ramp and tail:
        // >= 2^34 node-words (~0.5 ms at the LOP3 peak), e.g. C5's copy types; else it is bundled
        std::vector<uint64_t> work(jit_progs.size(), 0);
        std::vector<uint64_t> nodes_of(jit_progs.size(), 0);
        for (size_t i = 0; i < jit_progs.size(); ++i) nodes_of[i] = jit_progs[i].nodes.size() / 2;
        for (size_t w = 0; w < win_jit.size(); ++w)
            if (win_jit[w] >= 0) work[win_jit[w]] += nodes_of[win_jit[w]] * words_rank_of[w];
        uint64_t fill = 1ull << 34;
        if (const char *e = getenv("CEC_BUNDLE_BELOW")) fill = strtoull(e, nullptr, 10);
        const bool can_bundle = jcfg.splice && jcfg.sync_every > 0 && P->dwin.size() < (1u << 20) &&
                                getenv("CEC_NO_BUNDLE") == nullptr;
        uint32_t max_per = 24;
        uint64_t max_nodes = 24000;
        if (const char *e = getenv("CEC_BUNDLE_MAX")) max_per = std::max(1, atoi(e));
        std::vector<uint32_t> cur;
        uint64_t cur_nodes = 0;
        auto flush = [&]() {
            if (cur.empty()) return;
            for (uint32_t t = 0; t < cur.size(); ++t) {
                unit_of[cur[t]] = (uint32_t)units.size();
                sid_of[cur[t]] = t;
            }
            units.push_back(cur);
            cur.clear();
            cur_nodes = 0;
        };
        for (uint32_t i = 0; i < jit_progs.size(); ++i) {
            // large bodies (> 4096 ANDs, ~64 KB of SASS each) keep their own kernel: a bundle of
            // them would share one register allocation and spread SMs over several big bodies
            if (!can_bundle || work[i] >= fill || nodes_of[i] > 4096) {
                unit_of[i] = (uint32_t)units.size();
                sid_of[i] = 0;
                units.push_back({i});
                continue;
            }
            if (cur.size() >= max_per || cur_nodes + nodes_of[i] > max_nodes) flush();
            cur.push_back(i);
            cur_nodes += nodes_of[i];
        }
        flush();
    }
    std::vector<JitKernel *> kernels(units.size(), nullptr);
    // Block shape per compiled kernel: a large body (> 4096 ANDs, ~100 KB of SASS) runs as one
    // 512-thread block per SM whose 16 warps share instruction-cache lines (block-synchronous); a
    // small body fits the caches, and two 256-thread blocks per SM halve the warps that meet at each
    // pass barrier (C3: 4.67 -> 4.30 ms/step; C5's large types: 512 stays 10% faster).
    // CEC_JIT_THREADS / CEC_JIT_MINB override both.
    std::vector<JitConfig> ucfg(units.size(), jcfg);
    if (!getenv("CEC_JIT_THREADS") && !getenv("CEC_JIT_MINB") && jcfg.sync_every > 0)
        for (size_t u = 0; u < units.size(); ++u) {
            uint64_t mx = 0;
            for (uint32_t i : units[u]) mx = std::max<uint64_t>(mx, jit_progs[i].nodes.size() / 2);
            if (mx <= 4096) {
                ucfg[u].threads = 256;
                ucfg[u].min_blocks = 2;
                // a single small structure: static per-warp partition of its slices (no barriers, no
                // work-queue atomics). CEC_JIT_FREE=0 keeps the block-synchronous loop everywhere, =2
                // frees bundles too (C3 4.07 vs 3.91 ms: warps of one SM then run different bodies)
                const int fm = getenv("CEC_JIT_FREE") ? atoi(getenv("CEC_JIT_FREE")) : 1;
                ucfg[u].free_warps = jcfg.splice && (fm == 2 || (fm == 1 && units[u].size() == 1));
                if (ucfg[u].free_warps && units[u].size() == 1 && getenv("CEC_JIT_ILP"))
                    ucfg[u].ilp = std::max(1, std::min(2, atoi(getenv("CEC_JIT_ILP"))));
            }
        }
    P->jit_ms = 0.f;
    if (!units.empty()) {
        auto t0 = std::chrono::steady_clock::now();
        std::vector<std::string> errs(units.size());  // copied in the worker (messages are thread-local)
        const bool load = !c->host_only;
        std::vector<std::vector<const JitProgram *>> uprogs(units.size());
        for (size_t u = 0; u < units.size(); ++u)
            for (uint32_t i : units[u]) uprogs[u].push_back(&jit_progs[i]);
        // compile (CPU-heavy, thread-safe) in parallel without loading, then load serially
        c->workers().run((uint32_t)units.size(), [&](uint32_t i, unsigned) {
            const char *e = jit_get_unit(uprogs[i], ucfg[i], false, &kernels[i]);
            if (e) errs[i] = e;
        });
        for (size_t i = 0; i < units.size(); ++i) {
            if (!errs[i].empty()) return fail(c, CEC_E_CUDA, "JIT: %s", errs[i].c_str());
            if (load && !jit_kernel_loaded(kernels[i])) {  // cache hits of the first pass are loaded
                const char *e = jit_get_unit(uprogs[i], ucfg[i], true, &kernels[i]);
                if (e) return fail(c, CEC_E_CUDA, "JIT load: %s", e);
            }
        }
        P->jit_ms = std::chrono::duration<float, std::milli>(std::chrono::steady_clock::now() - t0).count();
    }
    auto lop3_of = [&](uint32_t w) -> uint64_t {
        const int32_t pi = win_jit[w];
        return pi >= 0 ? jit_kernel_lop3_sid(kernels[unit_of[pi]], sid_of[pi]) : P->win_nodes[w];
    };
    auto imad_of = [&](uint32_t w) -> uint64_t {
        const int32_t pi = win_jit[w];
        return pi >= 0 ? jit_kernel_imad_sid(kernels[unit_of[pi]], sid_of[pi]) : 0;
    };
    auto jwin = [&](uint32_t w) -> uint32_t {  // item window field: window | sid << 20 in bundles
        const int32_t pi = win_jit[w];
        return units[unit_of[pi]].size() > 1 ? (w | sid_of[pi] << 20) : w;
    };
    tm.lap("jit compile/cache");
    PhaseTimer tm2;
    P->jit_kernels = (uint32_t)units.size();
    P->jit_windows = 0;
    P->lop3_words = 0;
    P->imad_words = 0;
    for (uint32_t w = 0; w < win_jit.size(); ++w) {
        P->jit_windows += win_jit[w] >= 0;
        P->lop3_words += lop3_of(w) * words_rank_of[w];
        P->imad_words += imad_of(w) * words_rank_of[w];
    }
    // work items: slices of each window split into chunks; interpreter windows grouped by slot
    // budget, JIT windows by structure; largest windows first inside a group
    std::map<uint32_t, std::vector<uint32_t>> buckets;   // interpreter: slot budget -> windows
    std::map<int32_t, std::vector<uint32_t>> jgroups;    // JIT: compiled unit -> windows
    for (uint32_t w = 0; w < P->dwin.size(); ++w) {
        if (win_jit[w] >= 0) {
            jgroups[(int32_t)unit_of[win_jit[w]]].push_back(w);
            continue;
        }
        uint32_t b = (nslots_of[w] + 31) / 32 * 32;
        b = std::min(b, max_slot_cap);
        buckets[b].push_back(w);
    }
    // Each launch is a persistent grid pulling items; size items per GROUP so even a one-window
    // group (e.g. a bug-variant structure) splits into enough items to fill every SM.
    int cur_min_blocks = 1;  // the unit's configured blocks per SM (host-only plans: no occupancy query)
    std::string partition_err;
    auto add_items = [&](std::vector<uint32_t> ws, bool jit, LaunchGroup &g) {
        std::stable_sort(ws.begin(), ws.end(), [&](uint32_t a, uint32_t b) { return cost_of[a] > cost_of[b]; });
        g.nwin = (uint32_t)ws.size();
        for (uint32_t w : ws) {
            g.lop3_words += lop3_of(w) * words_rank_of[w];
            g.max_k = std::max(g.max_k, P->dwin[w].k);
            g.nodes = std::max(g.nodes, P->win_nodes[w]);
        }
        uint64_t group_slices = 0;
        for (uint32_t w : ws) {
            uint64_t ttw = tt_words_of(P->dwin[w].k), sb, se;
            win_range(w, (ttw + wps_of[w] - 1) / wps_of[w], &sb, &se);
            group_slices += se - sb;
        }
        const uint64_t target = (uint64_t)std::max(c->num_sms, 148) * 16 /*resident warps*/ * 8;
        uint64_t item_slices = std::min<uint64_t>(4096, std::max<uint64_t>(1, group_slices / target));
        if (jit && g.jit && jit_kernel_free(g.jit)) {
            // free warps: warp gw of the launch takes the contiguous slices [gw T / GW, (gw+1) T / GW)
            // of the group's concatenated (window, slice) space, cut into items at window ends
            const uint64_t wpb = (uint64_t)std::max(1, jit_kernel_block(g.jit) / 32);
            uint64_t blocks = (uint64_t)jit_kernel_blocks(g.jit, c->num_sms > 0 ? c->num_sms : 148, std::max(1, cur_min_blocks));
            blocks = std::max<uint64_t>(1, std::min(blocks, (group_slices + wpb - 1) / wpb));
            const uint64_t GW = blocks * wpb;
            g.free_blocks = (uint32_t)blocks;
            g.joff_off = (uint32_t)P->joff.size();
            std::vector<std::pair<uint32_t, uint64_t>> wl;  // (window, first slice) in group order
            std::vector<uint64_t> wstart{0};
            for (uint32_t w : ws) {
                uint64_t ttw = tt_words_of(P->dwin[w].k), sb, se;
                win_range(w, (ttw + wps_of[w] - 1) / wps_of[w], &sb, &se);
                if (se <= sb) continue;
                wl.push_back({w, sb});
                wstart.push_back(wstart.back() + (se - sb));
            }
            const size_t base = P->jitems.size();
            size_t wi = 0;
            for (uint64_t gw = 0; gw < GW; ++gw) {
                P->joff.push_back((uint32_t)(P->jitems.size() - base));
                uint64_t lo = gw * group_slices / GW;
                const uint64_t hi = (gw + 1) * group_slices / GW;
                while (lo < hi) {
                    while (wstart[wi + 1] <= lo) ++wi;
                    const uint64_t e = std::min(hi, wstart[wi + 1]);
                    const uint32_t w = wl[wi].first;
                    const uint64_t s0 = wl[wi].second + (lo - wstart[wi]);
                    P->jitems.push_back(JItem{jwin(w), (uint32_t)s0, (uint32_t)(s0 + (e - lo)), P->dwin[w].cmp_off});
                    lo = e;
                }
            }
            P->joff.push_back((uint32_t)(P->jitems.size() - base));
            // invariant: the items tile every window's slice range exactly once, in order
            std::vector<uint64_t> next(wl.size());
            for (size_t q = 0; q < wl.size(); ++q) next[q] = wl[q].second;
            size_t q = 0;
            for (size_t t = base; t < P->jitems.size(); ++t) {
                const JItem &it = P->jitems[t];
                while (q < wl.size() && jwin(wl[q].first) != it.win) ++q;
                if (q == wl.size() || it.s_begin != next[q] || it.s_end <= it.s_begin) {
                    partition_err = "free-warp partition does not tile the slice ranges";
                    return;
                }
                next[q] = it.s_end;
            }
            for (size_t r = 0; r < wl.size(); ++r)
                if (next[r] != wl[r].second + (wstart[r + 1] - wstart[r])) partition_err = "free-warp partition misses slices";
            return;
        }
        // block-synchronous JIT: an item is whole passes of one slice per warp of the kernel's block
        const uint64_t gpass = jit && g.jit ? (uint64_t)std::max(1, jit_slices_per_pass(g.jit)) : jit_pass;
        if (jit && gpass > 1) item_slices = std::max<uint64_t>(gpass, item_slices * gpass);
        for (uint32_t w : ws) {
            uint64_t ttw = tt_words_of(P->dwin[w].k), sb, se;
            win_range(w, (ttw + wps_of[w] - 1) / wps_of[w], &sb, &se);
            for (uint64_t s = sb; s < se; s += item_slices) {
                const uint32_t e = (uint32_t)std::min<uint64_t>(se, s + item_slices);
                if (jit)
                    P->jitems.push_back(JItem{jwin(w), (uint32_t)s, e, P->dwin[w].cmp_off});
                else
                    P->items.push_back(Item{w, (uint32_t)s, e, 0});
            }
        }
    };
    for (auto &kv : jgroups) {
        LaunchGroup g{};
        g.jit = kernels[kv.first];
        cur_min_blocks = ucfg[kv.first].min_blocks;
        g.item_off = (uint32_t)P->jitems.size();
        add_items(kv.second, true, g);
        if (!partition_err.empty()) return fail(c, CEC_E_STATE, "%s", partition_err.c_str());
        g.nitems = (uint32_t)(P->jitems.size() - g.item_off);
        P->groups.push_back(g);
    }
    for (auto &kv : buckets) {
        LaunchGroup g{};
        g.nslots = kv.first;
        g.item_off = (uint32_t)P->items.size();
        add_items(kv.second, false, g);
        g.nitems = (uint32_t)(P->items.size() - g.item_off);
        P->groups.push_back(g);
    }
    // biggest groups first so the small launches fill in behind them
    std::stable_sort(P->groups.begin(), P->groups.end(),
                     [](const LaunchGroup &a, const LaunchGroup &b) { return a.nitems > b.nitems; });
    tm2.lap("work items + launch groups");
    (void)stop;
    (void)local;
    return CEC_OK;
}

cec_status upload(cec_ctx *c, cec_plan *P) {
    if (c->host_only) return CEC_OK;
    DevPlan &d = P->d;
    const size_t ncmp = std::max<size_t>(1, P->cmps.size()), nwin = std::max<size_t>(1, P->dwin.size());
    // one device block: [wins | prog | items | jitems] (uploaded by one H2D from pinned staging)
    // then [first | bound | neq_cnt | item_ctr] (initialised on the device by the reset kernel)
    auto al = [](size_t x) { return (x + 255) / 256 * 256; };
    const size_t b_wins = sizeof(DevWin) * P->dwin.size(), b_prog = sizeof(uint4) * P->prog.size(),
                 b_items = sizeof(Item) * P->items.size(), b_jitems = sizeof(JItem) * P->jitems.size(),
                 b_joff = sizeof(uint32_t) * P->joff.size();
    size_t off = 0;
    const size_t o_wins = off; off += al(std::max<size_t>(b_wins, 1));
    const size_t o_prog = off; off += al(std::max<size_t>(b_prog, 1));
    const size_t o_items = off; off += al(std::max<size_t>(b_items, 1));
    const size_t o_jitems = off; off += al(std::max<size_t>(b_jitems, 1));
    const size_t o_joff = off; off += al(std::max<size_t>(b_joff, 1));
    const size_t up_bytes = off;
    const size_t o_first = off; off += al(sizeof(unsigned long long) * ncmp);
    const size_t o_bound = off; off += al(sizeof(unsigned long long) * nwin);
    const size_t o_neq = off; off += al(sizeof(uint32_t) * nwin);
    const size_t o_ctr = off; off += al(sizeof(uint32_t) * std::max<size_t>(1, P->groups.size()));
    PhaseTimer tu;
    if (!c->devpool) c->devpool = std::make_shared<DevPool>();
    P->pool = c->devpool;
    CUDA_TRY(c, P->pool->get(off, &P->arena, &P->arena_cap));
    tu.lap("upload: device block");
    char *base = (char *)P->arena;
    d.wins = (DevWin *)(base + o_wins);
    d.prog = (uint4 *)(base + o_prog);
    d.items = (Item *)(base + o_items);
    d.jitems = (JItem *)(base + o_jitems);
    d.joff = (uint32_t *)(base + o_joff);
    d.first = (unsigned long long *)(base + o_first);
    d.bound = (unsigned long long *)(base + o_bound);
    d.neq_cnt = (uint32_t *)(base + o_neq);
    d.item_ctr = (uint32_t *)(base + o_ctr);
    {
        void *hst = nullptr;
        CUDA_TRY(c, P->pool->staging(up_bytes, &hst));
        tu.lap("upload: staging wait/alloc");
        char *h = (char *)hst;
        if (b_wins) memcpy(h + o_wins, P->dwin.data(), b_wins);
        if (b_prog >= (4u << 20)) {  // large interpreter programs (C3: ~9 MB): copied by the worker pool
            const size_t chunk = 1u << 20, nch = (b_prog + chunk - 1) / chunk;
            const char *src = reinterpret_cast<const char *>(P->prog.data());
            c->workers().run((uint32_t)nch, [&](uint32_t i, unsigned) {
                const size_t o = (size_t)i * chunk;
                memcpy(h + o_prog + o, src + o, std::min(chunk, b_prog - o));
            });
        } else if (b_prog) {
            memcpy(h + o_prog, P->prog.data(), b_prog);
        }
        if (b_items) memcpy(h + o_items, P->items.data(), b_items);
        if (b_jitems) memcpy(h + o_jitems, P->jitems.data(), b_jitems);
        if (b_joff) memcpy(h + o_joff, P->joff.data(), b_joff);
        tu.lap("upload: staging copies");
        CUDA_TRY(c, h2d(base, h, o_joff + b_joff, c->stream));
        CUDA_TRY(c, P->pool->staged(c->stream));
        tu.lap("upload: h2d issue");
    }
    if (P->simt.E) {
        SimtPlan &S = P->simt;
        if (c->opts.workspace && sizeof(uint32_t) * (uint64_t)S.E * S.rows <= c->opts.workspace_bytes) {
            S.d_simt = (uint4 *)c->opts.workspace;  // 16-byte aligned: cudaMalloc / torch allocations
            S.simt_in_workspace = true;
        } else {
            CUDA_TRY(c, dev_alloc((void **)&S.d_simt, sizeof(uint32_t) * (size_t)S.E * S.rows));
        }
        CUDA_TRY(c, dev_alloc((void **)&S.d_inputs, sizeof(uint4) * std::max<size_t>(1, S.h_inputs.size())));
        CUDA_TRY(c, dev_alloc((void **)&S.d_nodes, sizeof(uint4) * std::max<size_t>(1, S.h_nodes.size())));
        CUDA_TRY(c, dev_alloc((void **)&S.d_pairs, sizeof(uint4) * std::max<size_t>(1, S.h_pairs.size())));
        CUDA_TRY(c, dev_alloc((void **)&S.d_ttw, sizeof(unsigned long long) * std::max<size_t>(1, S.h_ttw.size())));
        CUDA_TRY(c, h2d(S.d_inputs, S.h_inputs.data(), sizeof(uint4) * S.h_inputs.size(), c->stream));
        CUDA_TRY(c, h2d(S.d_nodes, S.h_nodes.data(), sizeof(uint4) * S.h_nodes.size(), c->stream));
        CUDA_TRY(c, h2d(S.d_pairs, S.h_pairs.data(), sizeof(uint4) * S.h_pairs.size(), c->stream));
        CUDA_TRY(c, h2d(S.d_ttw, S.h_ttw.data(), sizeof(unsigned long long) * S.h_ttw.size(), c->stream));
    }
    CUDA_TRY(c, event_create(&P->ev0));
    CUDA_TRY(c, event_create(&P->ev1));
    CUDA_TRY(c, event_create(&P->sev[0]));
    CUDA_TRY(c, event_create(&P->sev[1]));
    c->stats.h2d_bytes = sizeof(DevWin) * P->dwin.size() + sizeof(uint4) * P->prog.size() +
                         sizeof(Item) * P->items.size() + sizeof(JItem) * P->jitems.size() +
                         sizeof(uint32_t) * P->joff.size();
    P->uploaded = true;
    return CEC_OK;
}

void free_dev(cec_plan *P) {
    if (P->pool && P->arena) P->pool->put(P->arena, P->arena_cap);
    P->arena = nullptr;
    P->arena_cap = 0;
    P->pool.reset();
    P->d = DevPlan{};
    if (!P->simt.simt_in_workspace) dev_free(P->simt.d_simt);
    P->simt.simt_in_workspace = false;
    dev_free(P->simt.d_inputs);
    dev_free(P->simt.d_nodes);
    dev_free(P->simt.d_pairs);
    dev_free(P->simt.d_ttw);
    P->simt.d_simt = nullptr;
    P->simt.d_inputs = P->simt.d_nodes = P->simt.d_pairs = nullptr;
    P->simt.d_ttw = nullptr;
    event_destroy(P->ev0);
    event_destroy(P->ev1);
    event_destroy(P->sev[0]);
    event_destroy(P->sev[1]);
    P->ev0 = P->ev1 = P->sev[0] = P->sev[1] = nullptr;
    graph_destroy(P->graph);
    P->graph = P->graph_stream = nullptr;
}


bool lex_less(const std::vector<uint32_t> &a, const std::vector<uint32_t> &b) {
    return std::lexicographical_compare(a.begin(), a.end(), b.begin(), b.end());
}

std::vector<uint32_t> set_union(const std::vector<uint32_t> &a, const std::vector<uint32_t> &b) {
    std::vector<uint32_t> u;
    u.reserve(a.size() + b.size());
    std::set_union(a.begin(), a.end(), b.begin(), b.end(), std::back_inserter(u));
    return u;
}

double est_cost(uint64_t nodes, size_t k) { return (double)nodes * (double)(k <= 5 ? 32 : (1ull << std::min<size_t>(k, 62))); }

}  // namespace

cec_plan::~cec_plan() { free_dev(this); }

extern "C" {

}  // extern "C"

// a2-a5 of a global check: supports, trivial pairs, routing by k, compares, windows and merging.
// Open-addressing map uint64 -> uint32 for the routing of all pairs (one probe sequence per lookup,
// no node allocations: the routing loop was bound by std::unordered_map). Key ~0 is the empty mark.
struct FlatMap64 {
    std::vector<uint64_t> key;
    std::vector<uint32_t> val;
    size_t mask = 0;
    explicit FlatMap64(size_t n) {
        size_t cap = 16;
        while (cap < 2 * n) cap <<= 1;
        key.assign(cap, ~0ull);
        val.assign(cap, 0);
        mask = cap - 1;
    }
    // the value slot of `k` (inserted with value `dflt` if absent; *inserted says which)
    uint32_t *slot(uint64_t k, uint32_t dflt, bool *inserted) {
        uint64_t h = k + 0x9E3779B97F4A7C15ull;
        h = (h ^ (h >> 30)) * 0xBF58476D1CE4E5B9ull;
        h = (h ^ (h >> 27)) * 0x94D049BB133111EBull;
        for (size_t i = (h ^ (h >> 31)) & mask;; i = (i + 1) & mask) {
            if (key[i] == k) {
                *inserted = false;
                return &val[i];
            }
            if (key[i] == ~0ull) {
                key[i] = k;
                val[i] = dflt;
                *inserted = true;
                return &val[i];
            }
        }
    }
};

static cec_status plan_route(cec_ctx *c, uint32_t n, const uint32_t *la, const uint32_t *lb, cec_plan *P,
                             std::vector<WinHost> &wins, PhaseTimer &tm) {
    P->num_pairs = n;
    P->la.assign(la, la + n);
    P->lb.assign(lb, lb + n);
    P->pre_verdict.assign(n, CEC_UNDECIDED);
    P->pre_cex.assign(n, CEC_NO_CEX);
    P->k.assign(n, 0);
    P->pair_cmp.assign(n, -1);
    const uint32_t kmax = c->opts.k_max;
    // a2/a3: supports, trivial pairs, routing by k; identical (unordered) pairs share one compare
    FlatMap64 seen(n);  // unordered literal pair -> compare (key < ~0: literals < 2^32 - 1)
    // identical supports share a window: hash of S -> first window with that hash, then a chain
    // through win_next (exact compare below); no per-window allocation
    FlatMap64 by_support(n);
    std::vector<uint32_t> win_next;
    auto supp_hash = [](const std::vector<uint32_t> &S) {
        uint64_t h = 0x9E3779B97F4A7C15ull ^ S.size();
        for (uint32_t x : S) h = (h ^ x) * 0x100000001B3ull, h ^= h >> 29;
        return h;
    };
    std::vector<WinHost> wins0;
    for (uint32_t p = 0; p < n; ++p)
        if ((la[p] >> 1) >= c->N() || (lb[p] >> 1) >= c->N())
            return fail(c, CEC_E_ARG, "pair %u: literal out of range", p);
    // a2: structural supports of all pairs, in parallel (independent TFI walks, own scratch each)
    std::vector<std::vector<uint32_t>> supp(n);
    std::vector<uint64_t> cones(n, 0);
    // On a device context the supports come from the GPU (supp_gpu.cu: one launch per level over
    // the whole AIG, lists saturating at k_max + 1); only pairs above k_max (exact k) and the
    // cost-aware merge (which needs cone sizes) walk cones on the host.
    std::vector<uint8_t> need_walk(n, 1);
    // The cost-aware merge also needs each pair's cone size: the GPU walks those too (cone_sizes,
    // supp_gpu.cu; CEC_CONES_GPU=0 walks them on the host), cones too large for its shared memory
    // fall back to the host walk.
    const bool cost = c->opts.merge == CEC_MERGE_COST;
    bool cones_gpu = !getenv("CEC_CONES_GPU") || atoi(getenv("CEC_CONES_GPU")) != 0;
    bool gpu_supp = !c->host_only && (!cost || cones_gpu) && n >= 64 && c->N() >= (1u << 16);
    if (const char *e = getenv("CEC_SUPP_GPU")) gpu_supp = !c->host_only && (!cost || cones_gpu) && atoi(e) != 0;
    if (gpu_supp) {
        cec_status st = cec_ensure_device_aig(c);
        if (st != CEC_OK) return st;
        if (!c->devpool) c->devpool = std::make_shared<DevPool>();
        const uint32_t cap = std::min<uint32_t>(kmax, MAX_K_ENUM) + 1;  // k above either is routed away
        std::vector<uint2> roots(n);
        for (uint32_t p = 0; p < n; ++p) roots[p] = make_uint2(la[p] >> 1, lb[p] >> 1);
        std::vector<uint32_t> lists, cnt;
        uint32_t nl = 0;
        CUDA_TRY(c, gpu_supports(*c->devpool, c->d_f0, c->d_f1, c->d_level_ids, c->level_off, c->I, c->N(), cap, roots,
                                 lists, cnt, c->stream, &nl, &c->supp_table));
        std::vector<uint32_t> gcone;
        if (cost) CUDA_TRY(c, gpu_cones(*c->devpool, c->d_f0, c->d_f1, c->I, roots, gcone, c->stream));
        for (uint32_t p = 0; p < n; ++p)
            if (cnt[p] < cap && (!cost || gcone[p] != 0xFFFFFFFFu)) {
                supp[p].assign(lists.begin() + (size_t)p * cap, lists.begin() + (size_t)p * cap + cnt[p]);
                if (cost) cones[p] = gcone[p];
                need_walk[p] = 0;
            }
        tm.lap(cost ? "supports + cones (gpu)" : "supports (gpu)");
    }
    if (std::find(need_walk.begin(), need_walk.end(), (uint8_t)1) != need_walk.end()) {
        WorkPool &wp = c->workers();
        const unsigned nt = (unsigned)std::min<uint64_t>(wp.size() + 1, (n + 63) / 64);
        std::atomic<uint32_t> next{0};
        auto work = [&](unsigned tid) {
            Scratch &X = c->pool[tid];
            X.init(c->N());
            std::vector<uint32_t> &stamp = X.stamp, &st = X.stack;
            uint32_t &ep = X.epoch;
            // chunks of consecutive pairs per thread: pairs of one PO group share their cone, so a
            // thread walks the same (cache-resident) nodes again
            for (uint32_t p0; (p0 = next.fetch_add(64)) < n;)
            for (uint32_t p = p0; p < std::min(n, p0 + 64); ++p) {
                if (!need_walk[p]) continue;
                ep = X.next_epoch();
                auto &S = supp[p];
                uint64_t nodes = 0;
                st.clear();
                for (uint32_t r : {la[p] >> 1, lb[p] >> 1})
                    if (stamp[r] != ep) {
                        stamp[r] = ep;
                        st.push_back(r);
                    }
                while (!st.empty()) {
                    const uint32_t v = st.back();
                    st.pop_back();
                    if (v >= 1 && v <= c->I) {
                        S.push_back(v);
                        continue;
                    }
                    if (v == 0) continue;
                    ++nodes;
                    for (uint32_t f : {c->f0[v] >> 1, c->f1[v] >> 1})
                        if (stamp[f] != ep) {
                            stamp[f] = ep;
                            st.push_back(f);
                        }
                }
                std::sort(S.begin(), S.end());
                cones[p] = nodes;
            }
        };
        if (nt <= 1) {
            work(wp.size());
        } else {
            wp.run(nt, [&](uint32_t, unsigned tid) { work(tid); });
        }
    }
    tm.lap("supports");
    P->cmps.reserve(n);
    wins0.reserve(n);
    win_next.reserve(n);
    for (uint32_t p = 0; p < n; ++p) {
        std::vector<uint32_t> &S = supp[p];
        const uint64_t cone = cones[p];
        P->k[p] = (uint32_t)S.size();
        if (la[p] == lb[p]) {
            P->pre_verdict[p] = CEC_EQUIVALENT;
            continue;
        }
        if (la[p] == (lb[p] ^ 1u)) {
            P->pre_verdict[p] = CEC_NOT_EQUIVALENT;
            P->pre_cex[p] = 0;
            continue;
        }
        if (S.size() > kmax || S.size() > MAX_K_ENUM) {
            P->pre_verdict[p] = CEC_UNDECIDED;
            continue;
        }
        P->pre_verdict[p] = DECIDED_BY_SIM;
        const uint64_t key = (uint64_t)std::min(la[p], lb[p]) << 32 | std::max(la[p], lb[p]);
        bool fresh = false;
        uint32_t *cslot = seen.slot(key, (uint32_t)P->cmps.size(), &fresh);
        if (!fresh) {
            P->pair_cmp[p] = (int32_t)*cslot;
            continue;
        }
        const uint32_t ci = *cslot;
        P->pair_cmp[p] = (int32_t)ci;
        uint64_t sh = supp_hash(S);
        if (sh == ~0ull) sh = 0;  // the empty mark (a hash collision is resolved by the exact compare)
        uint32_t *head = by_support.slot(sh, UINT32_MAX, &fresh);
        uint32_t wi = UINT32_MAX;
        for (uint32_t x = *head; x != UINT32_MAX && wi == UINT32_MAX; x = win_next[x])
            if (wins0[x].inputs == S) wi = x;
        if (wi == UINT32_MAX) {
            win_next.push_back(*head);
            *head = (uint32_t)wins0.size();
            WinHost w;
            w.inputs = S;
            w.cmps.push_back(ci);
            w.est_nodes = cone;
            wins0.push_back(std::move(w));
        } else {
            WinHost &w = wins0[wi];
            w.cmps.push_back(ci);
            w.est_nodes = std::max<uint64_t>(w.est_nodes, cone);
        }
        Cmp cm;  // the pair's support moves into its compare (no copy)
        cm.la = la[p];
        cm.lb = lb[p];
        cm.S = std::move(S);
        P->cmps.push_back(std::move(cm));
    }
    tm.lap("routing: pairs -> windows");
    // a5: window merging: windows sorted lexicographically by input list.
    std::vector<uint32_t> order(wins0.size());
    for (uint32_t i = 0; i < order.size(); ++i) order[i] = i;
    std::stable_sort(order.begin(), order.end(),
                     [&](uint32_t a, uint32_t b) { return lex_less(wins0[a].inputs, wins0[b].inputs); });
    tm.lap("routing: lexicographic sort");
    // a merged window is enumerated like a single pair's: never more than MAX_K_ENUM inputs
    // (its slice indices are u32), whatever k_s / k_max the caller passed
    const uint32_t ks = std::min({c->opts.k_s, kmax, (uint32_t)MAX_K_ENUM});
    for (uint32_t oi : order) {
        WinHost &w = wins0[oi];
        if (!wins.empty() && c->opts.merge != CEC_MERGE_OFF) {
            WinHost &cur = wins.back();
            std::vector<uint32_t> U = set_union(cur.inputs, w.inputs);
            bool ok = U.size() <= ks;
            if (ok && c->opts.merge == CEC_MERGE_COST)
                ok = est_cost(cur.est_nodes + w.est_nodes, U.size()) <=
                     est_cost(cur.est_nodes, cur.inputs.size()) + est_cost(w.est_nodes, w.inputs.size());
            if (ok) {
                cur.inputs.swap(U);
                cur.cmps.insert(cur.cmps.end(), w.cmps.begin(), w.cmps.end());
                cur.est_nodes += w.est_nodes;
                continue;
            }
        }
        wins.push_back(std::move(w));
    }
    tm.lap("routing+merging");
    return CEC_OK;
}

extern "C" {

cec_status cec_plan_exhaustive(cec_ctx *c, uint32_t n, const uint32_t *la, const uint32_t *lb, cec_plan **out) {
    PhaseTimer tm;
    if (!c || !out || (n && (!la || !lb))) return fail(c, CEC_E_ARG, "null argument");
    *out = nullptr;
    auto t0 = std::chrono::steady_clock::now();
    std::unique_ptr<cec_plan> P(new (std::nothrow) cec_plan());
    if (!P) return CEC_E_NOMEM;
    std::vector<WinHost> wins;
    cec_status st = plan_route(c, n, la, lb, P.get(), wins, tm);
    if (st != CEC_OK) return st;
    st = finish_plan(c, P.get(), wins, nullptr, false);
    if (st != CEC_OK) return st;
    tm.lap("finish_plan");
    auto t1 = std::chrono::steady_clock::now();
    P->host_ms = std::chrono::duration<float, std::milli>(t1 - t0).count();
    c->stats.host_prep_ms = P->host_ms;
    c->stats.node_patterns = P->W_rank;
    c->stats.node_patterns_all = P->W_all;
    c->stats.num_windows = (uint32_t)P->dwin.size();
    c->stats.jit_ms = P->jit_ms;
    c->stats.jit_kernels = P->jit_kernels;
    c->stats.jit_windows = P->jit_windows;
    c->stats.lop3_words = P->lop3_words;
    c->stats.imad_words = P->imad_words;
    st = upload(c, P.get());
    if (st != CEC_OK) {
        free_dev(P.get());
        return st;
    }
    tm.lap("upload");
    *out = P.release();
    return CEC_OK;
}

cec_status cec_plan_run(cec_ctx *c, cec_plan *P) {
    if (!c || !P) return CEC_E_ARG;
    if (c->host_only) return fail(c, CEC_E_CUDA, "host-only context: no CUDA device (no CPU fallback)");
    if (!P->uploaded) return fail(c, CEC_E_STATE, "plan not uploaded");
    uint32_t nl = 0;
    const char *e = nullptr;
    // a plan that is run again is replayed as a CUDA graph (captured on its second run)
    // (host-barrier emulation synchronises inside the run: no graph capture)
    const bool use_graph = !P->simt.E && P->runs >= 1 && getenv("CEC_NO_GRAPH") == nullptr &&
                           getenv("CEC_PROFILE_GROUPS") == nullptr && !(c->peer.on && c->peer.host_barrier);
    // a10 over peer memory (peer.cu) when cec_peer_import connected this rank; else NCCL below
    const bool peer = c->peer.on && !P->simt.E;
    PeerRun pr;
    if (peer) {
        if (P->cmps.size() > c->peer.cap_cmp || P->dwin.size() > c->peer.cap_win)
            return fail(c, CEC_E_ARG, "plan exceeds the peer exchange capacity (%u compares, %u windows)",
                        c->peer.cap_cmp, c->peer.cap_win);
        pr = peer_run_of(c->peer, P->d.first);
    }
    if (use_graph && P->graph && (P->graph_stream != c->stream || P->graph_peer_gen != c->peer.gen)) {
        graph_destroy(P->graph);
        P->graph = nullptr;
    }
    if (use_graph && !P->graph) {
        e = graph_capture_run(P->d, P->groups, (uint32_t)P->dwin.size(), (uint32_t)P->cmps.size(), c->stream,
                              c->num_sms, &P->graph_launches, &c->aux, &P->graph, peer ? &pr : nullptr,
                              P->sweep_timing ? P->sev : nullptr);
        P->graph_stream = c->stream;
        P->graph_peer_gen = c->peer.gen;
        if (e) return fail(c, CEC_E_CUDA, "CUDA: %s (graph capture)", e);
    }
    CUDA_TRY(c, event_record(P->ev0, c->stream));
    if (use_graph) {
        e = graph_launch(P->graph, c->stream);
        nl = P->graph_launches;
    } else {
        e = P->simt.E ? launch_simt(P->simt, P->d.first, (uint32_t)P->cmps.size(), c->stream, c->num_sms, &nl)
                      : launch_run(P->d, P->groups, (uint32_t)P->dwin.size(), (uint32_t)P->cmps.size(), c->stream,
                                   c->num_sms, &nl, &c->aux, peer ? &pr : nullptr,
                                   P->no_join && !c->comm && !peer, P->sweep_timing ? P->sev : nullptr);
    }
    if (e) return fail(c, CEC_E_CUDA, "CUDA: %s (kernel launch)", e);
    P->sweep_timed_last = P->sweep_timing && !P->simt.E;
    if (c->comm && !peer && !P->cmps.empty()) {  // a10: one NCCL min all-reduce of first_idx
        ncclResult_t r = g_nccl.all_reduce(P->d.first, P->d.first, P->cmps.size(), ncclUint64, ncclMin, c->comm,
                                           (cudaStream_t)c->stream);
        if (r != ncclSuccess) return fail(c, CEC_E_NCCL, "NCCL: %s", g_nccl.err(r));
    }
    CUDA_TRY(c, event_record(P->ev1, c->stream));
    c->stats.num_launches = nl;
    c->stats.node_patterns = P->W_rank;
    c->stats.node_patterns_all = P->W_all;
    c->stats.num_windows = (uint32_t)P->dwin.size();
    c->stats.max_k = P->max_k;
    c->stats.max_slots = P->max_slots;
    c->stats.imad_words = P->imad_words;
    c->stats.lop3_words = P->lop3_words;  // this run's algorithmic LOP3 words (local checks included)
    c->stats.jit_windows = P->jit_windows;
    c->stats.jit_kernels = P->jit_kernels;
    P->ran = true;
    ++P->runs;
    return CEC_OK;
}

}  // extern "C"
static void resolve_results(cec_ctx *c, cec_plan *P, const std::vector<unsigned long long> &first, int32_t *verdict,
                            uint64_t *cex, uint32_t *k_out);
extern "C" {

cec_status cec_plan_results(cec_ctx *c, cec_plan *P, int32_t *verdict, uint64_t *cex, uint32_t *k_out) {
    if (!c || !P || (P->num_pairs && !verdict)) return fail(c, CEC_E_ARG, "null argument");
    std::vector<unsigned long long> first(P->cmps.size(), ~0ull);
    if (!P->cmps.empty()) {
        if (!P->ran) return fail(c, CEC_E_STATE, "plan has not been run");
        CUDA_TRY(c, d2h(first.data(), P->d.first, sizeof(unsigned long long) * first.size(), c->stream));
    }
    c->stats.d2h_bytes = sizeof(unsigned long long) * first.size();
    if (P->ran) {
        CUDA_TRY(c, stream_sync(c->stream));
        if (peer_failed(c)) return fail(c, CEC_E_NCCL, "peer barrier timed out (a peer rank never arrived)");
        float ms = 0.f;
        CUDA_TRY(c, event_elapsed(&ms, P->ev0, P->ev1));
        c->stats.kernel_ms = ms;
    }
    resolve_results(c, P, first, verdict, cex, k_out);
    return CEC_OK;
}

}  // extern "C"

// a11: per user pair, verdict and own-order CEX (pext of the merged index) from first[cmp].
static void resolve_results(cec_ctx *c, cec_plan *P, const std::vector<unsigned long long> &first, int32_t *verdict,
                            uint64_t *cex, uint32_t *k_out) {
    if (!P->local) {
        c->last_verdict.assign(P->num_pairs, CEC_UNDECIDED);
        c->last_cex.assign(P->num_pairs, CEC_NO_CEX);
        c->last_support.assign(P->num_pairs, {});
    }
    for (uint32_t p = 0; p < P->num_pairs; ++p) {
        int32_t v = P->pre_verdict[p];
        uint64_t x = P->pre_cex[p];
        if (v == DECIDED_BY_SIM) {
            const Cmp &cm = P->cmps[P->pair_cmp[p]];
            const unsigned long long f = first[P->pair_cmp[p]];
            if (P->local) {
                v = f == ~0ull ? CEC_EQUIVALENT : CEC_UNDECIDED;  // a12: mismatch may be an SDC
                x = CEC_NO_CEX;
            } else if (f == ~0ull) {
                v = CEC_EQUIVALENT;
                x = CEC_NO_CEX;
            } else {
                v = CEC_NOT_EQUIVALENT;
                x = cec_pext64(f, cm.ownmask);  // a11: merged index -> own index (Q8)
            }
        }
        verdict[p] = v;
        if (cex) cex[p] = x;
        if (k_out) k_out[p] = P->k[p];
        if (!P->local) {
            c->last_verdict[p] = v;
            c->last_cex[p] = x;
            // cec_get_cex maps bit j of the own index to the j-th support PI: a simulated pair's
            // compare holds exactly that sorted support (no second TFI walk); a pair refuted
            // without simulation (lit_a == lit_b ^ 1) has index 0, i.e. every PI 0
            if (v == CEC_NOT_EQUIVALENT && P->pre_verdict[p] == DECIDED_BY_SIM)
                c->last_support[p] = P->cmps[P->pair_cmp[p]].S;
        }
    }
    if (!P->local) c->have_last = true;
}

extern "C" {

cec_status cec_plan_sweep_timing(cec_plan *P, int on) {
    if (!P) return CEC_E_ARG;
    if (P->sweep_timing != (on != 0) && P->graph) {  // the captured run has (no) event nodes: recapture
        graph_destroy(P->graph);
        P->graph = nullptr;
    }
    P->sweep_timing = on != 0;
    return CEC_OK;
}

cec_status cec_plan_sweep_ms(const cec_plan *P, float *ms) {
    if (!P || !ms) return CEC_E_ARG;
    if (!P->ran || !P->sweep_timed_last || P->simt.E || !P->sev[0] || !P->sev[1] || P->no_join) return CEC_E_STATE;
    const char *e = event_elapsed(ms, P->sev[0], P->sev[1]);  // fails if the run has not completed
    return e ? CEC_E_STATE : CEC_OK;
}

cec_status cec_plan_info(const cec_plan *P, uint32_t *nw, uint64_t *W, uint32_t *mk, uint32_t *ms) {
    if (!P) return CEC_E_ARG;
    if (nw) *nw = (uint32_t)P->dwin.size();
    if (W) *W = P->W_all;
    if (mk) *mk = P->max_k;
    if (ms) *ms = P->max_slots;
    return CEC_OK;
}

cec_status cec_plan_window(const cec_plan *P, uint32_t w, uint32_t *inputs, uint32_t *k, uint32_t *nn,
                           uint32_t *pairs, uint32_t *np) {
    if (!P || w >= P->dwin.size()) return CEC_E_ARG;
    if (k) *k = (uint32_t)P->win_inputs[w].size();
    if (inputs)
        for (size_t j = 0; j < P->win_inputs[w].size(); ++j) inputs[j] = P->win_inputs[w][j];
    if (nn) *nn = P->win_nodes[w];
    // user pairs whose compare lives in window w
    uint32_t cnt = 0;
    const DevWin &dw = P->dwin[w];
    for (uint32_t p = 0; p < P->num_pairs; ++p) {
        int32_t ci = P->pair_cmp[p];
        if (ci >= (int32_t)dw.cmp_off && ci < (int32_t)(dw.cmp_off + dw.ncmp)) {
            if (pairs) pairs[cnt] = p;
            ++cnt;
        }
    }
    if (np) *np = cnt;
    return CEC_OK;
}

void cec_plan_free(cec_plan *P) {
    if (!P) return;
    free_dev(P);
    delete P;
}

cec_status cec_sim_exhaustive(cec_ctx *c, uint32_t n, const uint32_t *la, const uint32_t *lb, int32_t *verdict,
                              uint64_t *cex, uint32_t *k_out) {
    if (!c) return CEC_E_ARG;
    if (c->host_only) return fail(c, CEC_E_CUDA, "host-only context: no CUDA device (no CPU fallback)");
    if (n && (!la || !lb || !verdict)) return fail(c, CEC_E_ARG, "null argument");
    PhaseTimer tm;
    auto t0 = std::chrono::steady_clock::now();
    std::unique_ptr<cec_plan> P(new (std::nothrow) cec_plan());
    if (!P) return CEC_E_NOMEM;
    std::vector<WinHost> wins;
    cec_status st = plan_route(c, n, la, lb, P.get(), wins, tm);
    if (st != CEC_OK) return st;
    // Pipelined execution: the merged windows are cut into K chunks; chunk i is planned (node
    // orders, programs, work items), uploaded and launched while the GPU still runs chunk i-1, so
    // the host's per-window planning hides behind the sweep. Each chunk is an independent sub-plan
    // (own compares, bounds, launch groups); results are gathered per compare at the end.
    // It pays when the sweep dominates per-window planning (median window k >= 20, e.g. C5); with
    // many small windows (C3) chunking only fragments the launch groups.
    int K = 1;
    if (!wins.empty()) {
        std::vector<uint32_t> ks(wins.size());
        for (size_t w = 0; w < wins.size(); ++w) ks[w] = (uint32_t)wins[w].inputs.size();
        std::nth_element(ks.begin(), ks.begin() + ks.size() / 2, ks.end());
        if (ks[ks.size() / 2] >= 20) K = 4;
    }
    if (const char *e = getenv("CEC_PIPELINE")) K = std::max(1, atoi(e));
    if (c->opts.engine == CEC_ENGINE_SIMT || wins.size() < (size_t)2 * K) K = 1;
    std::vector<double> wcost(wins.size());
    double total = 0;
    for (size_t w = 0; w < wins.size(); ++w) {
        const uint32_t k = (uint32_t)std::min<size_t>(wins[w].inputs.size(), 40);
        wcost[w] = std::ldexp(1.0, (int)k) * (double)(1 + std::max<uint64_t>(wins[w].est_nodes, wins[w].cmps.size()));
        total += wcost[w];
    }
    // Many small windows (C3: median k < 20, thousands of windows): geometric chunks would only
    // fragment the bundle kernels, but the sweep is still dominated by a few large windows. Those
    // (estimated sweep >= 2^26 node-words) form a first chunk that is planned and launched alone;
    // the GPU runs them while the host plans the rest
    // (bundles and interpreter windows). CEC_PIPE_SPLIT = the node-word threshold (0 = off); C3:
    // 154 of 3253 windows carry 95% of the sweep at 2^26, and the call takes 15.6-16.3 ms instead
    // of 18.4-18.6 (2^24: 16.1, 2^28: 16.5, 2^30: 17.3-18.9; profiles/round2s2_c3_split_sweep.txt).
    std::vector<size_t> cut{0};
    double split_nw = std::ldexp(1.0, 26);
    if (const char *e = getenv("CEC_PIPE_SPLIT")) split_nw = atof(e);
    size_t split_min = 256;  // windows; CEC_PIPE_SPLIT_MINWIN
    if (const char *e = getenv("CEC_PIPE_SPLIT_MINWIN")) split_min = strtoull(e, nullptr, 10);
    bool split = false;
    if (getenv("CEC_PIPE_SPLIT_DEBUG"))
        for (int e = 20; e <= 38; e += 2) {
            size_t nb = 0;
            double bc = 0;
            for (size_t w = 0; w < wins.size(); ++w)
                if (wcost[w] / 32.0 >= std::ldexp(1.0, e)) ++nb, bc += wcost[w];
            fprintf(stderr, "[cec] split 2^%d: %zu of %zu windows, %.3f of the cost\n", e, nb, wins.size(), bc / total);
        }
    if (K == 1 && split_nw > 0 && wins.size() >= split_min && c->opts.engine != CEC_ENGINE_SIMT) {
        std::vector<uint8_t> big(wins.size(), 0);
        size_t nbig = 0;
        double big_cost = 0;
        for (size_t w = 0; w < wins.size(); ++w)
            if (wcost[w] / 32.0 >= split_nw) big[w] = 1, ++nbig, big_cost += wcost[w];
        // worth it only when the first chunk is a small share of the windows and carries most of
        // the sweep (its kernels then cover the planning of everything else)
        if (nbig > 0 && nbig * 8 <= wins.size() && big_cost >= 0.5 * total) {
            std::vector<WinHost> reord;
            std::vector<double> rc;
            reord.reserve(wins.size());
            for (int pass = 0; pass < 2; ++pass)
                for (size_t w = 0; w < wins.size(); ++w)
                    if (big[w] == (pass == 0)) reord.push_back(std::move(wins[w])), rc.push_back(wcost[w]);
            wins.swap(reord);
            wcost.swap(rc);
            cut.push_back(nbig);
            split = true;
            char what[64];
            snprintf(what, sizeof what, "call: split %zu big of %zu", nbig, wins.size());
            tm.lap(what);
        }
    }
    // contiguous window ranges growing geometrically (4%, 8%, 16%, ... of the cost): the GPU starts
    // after planning a small first chunk, and each chunk's kernels (~2x the host time to plan the
    // same windows) cover the planning of the next, twice as large, chunk
    if (!split) {
        double first = 0.04, growth = 2.0;  // tunable: CEC_PIPE_FIRST (fraction), CEC_PIPE_GROWTH
        if (const char *e = getenv("CEC_PIPE_FIRST")) first = std::max(1e-4, atof(e));
        if (const char *e = getenv("CEC_PIPE_GROWTH")) growth = std::max(1.0, atof(e));
        double acc = 0, chunk = K > 1 ? first * total : total, target = chunk;
        for (size_t w = 0; w < wins.size(); ++w) {
            acc += wcost[w];
            if (K > 1 && acc >= target && w + 1 < wins.size()) {
                cut.push_back(w + 1);
                chunk *= growth;
                target = acc + chunk;
            }
        }
    }
    cut.push_back(wins.size());
    struct Sub {
        std::unique_ptr<cec_plan> p;
        std::vector<uint32_t> gcmp;  // local compare j (before finish_plan's renumbering) -> global
    };
    std::vector<Sub> subs;
    cec_stats agg{};
    float jit_ms = 0.f;
    for (size_t ch = 0; ch + 1 < cut.size(); ++ch) {
        if (cut[ch] == cut[ch + 1]) continue;
        Sub S;
        S.p.reset(new (std::nothrow) cec_plan());
        if (!S.p) return CEC_E_NOMEM;
        std::vector<WinHost> cw;
        // the chunk takes the windows' inputs and the compares' supports by move (each window /
        // compare belongs to one chunk); the supports move back at the gather
        for (size_t w = cut[ch]; w < cut[ch + 1]; ++w) {
            WinHost h;
            h.inputs = std::move(wins[w].inputs);
            h.est_nodes = wins[w].est_nodes;
            for (uint32_t ci : wins[w].cmps) {
                h.cmps.push_back((uint32_t)S.gcmp.size());
                S.gcmp.push_back(ci);
                S.p->cmps.push_back(std::move(P->cmps[ci]));
            }
            cw.push_back(std::move(h));
        }
        S.p->pair_cmp.resize(S.gcmp.size());
        for (uint32_t j = 0; j < S.gcmp.size(); ++j) S.p->pair_cmp[j] = (int32_t)j;
        if ((st = finish_plan(c, S.p.get(), cw, nullptr, false)) != CEC_OK) return st;
        // chunks before the last do not join the side streams: the next chunk's kernels start while
        // this chunk's tails drain (the last chunk's join, in stream order, covers them all)
        S.p->no_join = ch + 2 < cut.size() && getenv("CEC_PIPE_JOIN") == nullptr;
        if ((st = upload(c, S.p.get())) != CEC_OK) {
            free_dev(S.p.get());
            return st;
        }
        tm.lap("call: chunk upload");
        if (!S.p->cmps.empty() && (st = cec_plan_run(c, S.p.get())) != CEC_OK) {
            free_dev(S.p.get());
            return st;
        }
        tm.lap("call: chunk launch");
        agg.num_launches += c->stats.num_launches;
        agg.node_patterns += S.p->W_rank;
        agg.node_patterns_all += S.p->W_all;
        agg.num_windows += (uint32_t)S.p->dwin.size();
        agg.max_k = std::max(agg.max_k, S.p->max_k);
        agg.max_slots = std::max(agg.max_slots, S.p->max_slots);
        agg.jit_kernels += S.p->jit_kernels;
        agg.jit_windows += S.p->jit_windows;
        agg.lop3_words += S.p->lop3_words;
        agg.imad_words += S.p->imad_words;
        agg.h2d_bytes += c->stats.h2d_bytes;
        jit_ms += S.p->jit_ms;
        subs.push_back(std::move(S));
    }
    P->host_ms = std::chrono::duration<float, std::milli>(std::chrono::steady_clock::now() - t0).count();
    tm.lap("call: plan+launch (pipelined)");
    // gather: first[] of every chunk into the global compare order, with the chunk's pext masks
    std::vector<unsigned long long> first(P->cmps.size(), ~0ull);
    std::vector<std::vector<unsigned long long>> part(subs.size());
    for (size_t i = 0; i < subs.size(); ++i) {
        part[i].assign(subs[i].p->cmps.size(), ~0ull);
        if (!part[i].empty()) {
            cec_status s2 = CEC_OK;
            const char *e = d2h(part[i].data(), subs[i].p->d.first, sizeof(unsigned long long) * part[i].size(), c->stream);
            if (e) s2 = fail(c, CEC_E_CUDA, "CUDA: %s", e);
            if (s2 != CEC_OK) {
                for (auto &x : subs) free_dev(x.p.get());
                return s2;
            }
        }
    }
    const char *se = stream_sync(c->stream);
    tm.lap("call: wait for the GPU");
    if (!se && peer_failed(c)) {
        for (auto &x : subs) free_dev(x.p.get());
        return fail(c, CEC_E_NCCL, "peer barrier timed out (a peer rank never arrived)");
    }
    float kms = 0.f;
    if (!se && !subs.empty() && subs.front().p->ran && subs.back().p->ran)
        se = event_elapsed(&kms, subs.front().p->ev0, subs.back().p->ev1);
    for (size_t i = 0; i < subs.size(); ++i) {
        const Sub &S = subs[i];
        for (uint32_t j = 0; j < S.gcmp.size(); ++j) {
            const int32_t lj = S.p->pair_cmp[j];  // finish_plan's renumbering of local compare j
            P->cmps[S.gcmp[j]].ownmask = S.p->cmps[lj].ownmask;
            P->cmps[S.gcmp[j]].S = std::move(S.p->cmps[lj].S);
            first[S.gcmp[j]] = part[i][lj];
        }
        free_dev(S.p.get());
    }
    if (se) return fail(c, CEC_E_CUDA, "CUDA: %s", se);
    tm.lap("call: gather + free chunks");
    resolve_results(c, P.get(), first, verdict, cex, k_out);
    tm.lap("call: resolve results");
    const float host_ms = P->host_ms;
    c->stats.num_launches = agg.num_launches;
    c->stats.node_patterns = agg.node_patterns;
    c->stats.node_patterns_all = agg.node_patterns_all;
    c->stats.num_windows = agg.num_windows;
    c->stats.max_k = agg.max_k;
    c->stats.max_slots = agg.max_slots;
    c->stats.jit_kernels = agg.jit_kernels;
    c->stats.jit_windows = agg.jit_windows;
    c->stats.lop3_words = agg.lop3_words;
    c->stats.imad_words = agg.imad_words;
    c->stats.h2d_bytes = agg.h2d_bytes;
    c->stats.d2h_bytes = sizeof(unsigned long long) * first.size();
    c->stats.jit_ms = jit_ms;
    c->stats.kernel_ms = kms;
    c->stats.host_prep_ms = host_ms;
    tm.lap("call: stats + return");
    return CEC_OK;
}

static cec_status sim_signatures(cec_ctx *c, uint32_t W, uint64_t seed, const uint32_t *pi_words, uint64_t *sig_out,
                                 uint8_t *phase_out);

cec_status cec_ensure_device_aig(cec_ctx *c) {
    if (c->host_only) return fail(c, CEC_E_CUDA, "host-only context");
    const uint32_t N = c->N();
    if (!c->d_aig_valid) {  // AIG and level CSR on the device (a1)
        uint32_t maxl = 0;
        for (uint32_t id = 0; id < N; ++id) maxl = std::max(maxl, c->level[id]);
        c->level_off.assign(maxl + 2, 0);
        for (uint32_t id = 1 + c->I; id < N; ++id) ++c->level_off[c->level[id] + 1];
        for (size_t l = 1; l < c->level_off.size(); ++l) c->level_off[l] += c->level_off[l - 1];
        std::vector<uint32_t> ids(std::max<uint32_t>(1, c->A)), fill(c->level_off.begin(), c->level_off.end());
        for (uint32_t id = 1 + c->I; id < N; ++id) ids[fill[c->level[id]]++] = id;
        if (!c->d_f0 || c->d_aig_cap < N) {  // (re)allocate; ids.size() <= N
            dev_free(c->d_f0);
            dev_free(c->d_f1);
            dev_free(c->d_level_ids);
            c->d_f0 = c->d_f1 = c->d_level_ids = nullptr;
            c->d_aig_cap = 0;
            CUDA_TRY(c, dev_alloc((void **)&c->d_f0, sizeof(uint32_t) * N));
            CUDA_TRY(c, dev_alloc((void **)&c->d_f1, sizeof(uint32_t) * N));
            CUDA_TRY(c, dev_alloc((void **)&c->d_level_ids, sizeof(uint32_t) * N));
            c->d_aig_cap = N;
        }
        CUDA_TRY(c, h2d(c->d_f0, c->f0.data(), sizeof(uint32_t) * N, c->stream));
        CUDA_TRY(c, h2d(c->d_f1, c->f1.data(), sizeof(uint32_t) * N, c->stream));
        CUDA_TRY(c, h2d(c->d_level_ids, ids.data(), sizeof(uint32_t) * ids.size(), c->stream));
        CUDA_TRY(c, stream_sync(c->stream));
        c->d_aig_valid = true;
    }
    return CEC_OK;
}

cec_status cec_sim_random(cec_ctx *c, uint32_t W, uint64_t seed, uint64_t *sig_out, uint8_t *phase_out) {
    return sim_signatures(c, W, seed, nullptr, sig_out, phase_out);
}

cec_status cec_sim_patterns(cec_ctx *c, uint32_t W, const uint32_t *pi_words, uint64_t *sig_out, uint8_t *phase_out) {
    if (!pi_words) return fail(c, CEC_E_ARG, "null pi_words");
    return sim_signatures(c, W, 0, pi_words, sig_out, phase_out);
}

static cec_status sim_signatures(cec_ctx *c, uint32_t W, uint64_t seed, const uint32_t *pi_words, uint64_t *sig_out,
                                 uint8_t *phase_out) {
    if (!c || !sig_out || W == 0) return fail(c, CEC_E_ARG, "null argument or num_words == 0");
    if (c->host_only) return fail(c, CEC_E_CUDA, "host-only context: no CUDA device (no CPU fallback)");
    const uint32_t N = c->N();
    {
        cec_status st = cec_ensure_device_aig(c);
        if (st != CEC_OK) return st;
    }
    uint32_t *tt = nullptr;
    unsigned long long *sig = nullptr;
    uint8_t *ph = nullptr;
    struct Guard {
        void **p[3];
        ~Guard() {
            for (auto q : p) dev_free(*q);
        }
    } guard{{(void **)&tt, (void **)&sig, (void **)&ph}};
    CUDA_TRY(c, dev_alloc((void **)&tt, sizeof(uint32_t) * (size_t)N * W));
    CUDA_TRY(c, dev_alloc((void **)&sig, sizeof(unsigned long long) * N));
    CUDA_TRY(c, dev_alloc((void **)&ph, N));
    uint32_t nl = 0;
    if (pi_words) {  // caller patterns: PI id i+1 takes words pi_words[i*W .. i*W+W)
        CUDA_TRY(c, dev_memset(tt, 0, sizeof(uint32_t) * W, c->stream));
        CUDA_TRY(c, h2d(tt + W, pi_words, sizeof(uint32_t) * (size_t)c->I * W, c->stream));
    }
    const char *e = random_sim(c->d_f0, c->d_f1, c->d_level_ids, c->level_off, c->I, N, W, seed, tt, sig, ph, c->stream,
                               c->num_sms, &nl, pi_words != nullptr);
    if (e) return fail(c, CEC_E_CUDA, "CUDA: %s (random simulation)", e);
    CUDA_TRY(c, d2h(sig_out, sig, sizeof(unsigned long long) * N, c->stream));
    std::vector<uint8_t> phase(N);
    CUDA_TRY(c, d2h(phase.data(), ph, N, c->stream));
    CUDA_TRY(c, stream_sync(c->stream));
    if (phase_out) std::memcpy(phase_out, phase.data(), N);
    return CEC_OK;
}

cec_status cec_get_cex(cec_ctx *c, uint32_t p, uint8_t *pis) {
    if (!c || !pis) return CEC_E_ARG;
    if (!c->have_last) return fail(c, CEC_E_STATE, "no global check has been run");
    if (p >= c->last_verdict.size()) return fail(c, CEC_E_ARG, "pair index out of range");
    if (c->last_verdict[p] != CEC_NOT_EQUIVALENT) return fail(c, CEC_E_NOCEX, "pair %u is not NOT_EQUIVALENT", p);
    std::memset(pis, 0, c->I);
    const auto &S = c->last_support[p];
    const uint64_t x = c->last_cex[p];
    for (size_t j = 0; j < S.size() && j < 64; ++j) pis[S[j] - 1] = (uint8_t)((x >> j) & 1u);
    return CEC_OK;
}

cec_status cec_check_local_cuts(cec_ctx *c, uint32_t n, const uint32_t *la, const uint32_t *lb,
                                const uint32_t *cut_off, const uint32_t *leaves, int32_t *verdict) {
    if (!c || (n && (!la || !lb || !cut_off || !verdict))) return fail(c, CEC_E_ARG, "null argument");
    if (c->host_only) return fail(c, CEC_E_CUDA, "host-only context: no CUDA device (no CPU fallback)");
    std::unique_ptr<cec_plan> P;
    uint32_t bad = 0, first_bad = 0;
    cec_status st = local_checks_launch(c, n, la, lb, cut_off, leaves, P, &bad, &first_bad);
    if (st != CEC_OK) return st;
    st = local_checks_collect(c, P.get(), verdict);
    if (st != CEC_OK) return st;
    if (bad) return fail(c, CEC_E_CUT, "check %u: leaves are not a cut of the pair (%u bad checks)", first_bad, bad);
    return CEC_OK;
}

}  // extern "C"

// a12 split in two so a caller can overlap host work with the checks on the GPU (the Alg. 2 pass
// of cuts.cpp flushes its common-cut buffer through these): validate + plan + upload + launch
// (asynchronous on the context stream), then collect (wait, read back, free the device block).
cec_status local_checks_launch(cec_ctx *c, uint32_t n, const uint32_t *la, const uint32_t *lb, const uint32_t *cut_off,
                               const uint32_t *leaves, std::unique_ptr<cec_plan> &out, uint32_t *bad_out,
                               uint32_t *first_bad_out, bool trusted_cuts) {
    auto t0 = std::chrono::steady_clock::now();
    std::unique_ptr<cec_plan> P(new (std::nothrow) cec_plan());
    if (!P) return CEC_E_NOMEM;
    P->local = true;
    P->num_pairs = n;
    P->pre_verdict.assign(n, CEC_UNDECIDED);
    P->pre_cex.assign(n, CEC_NO_CEX);
    P->k.assign(n, 0);
    P->pair_cmp.assign(n, -1);
    const uint32_t kcap = std::min<uint32_t>(c->opts.k_max, 24);
    std::vector<WinHost> wins;
    std::vector<uint32_t> stop(c->N(), 0);
    uint32_t bad = 0, first_bad = 0;
    uint32_t sep = 0;
    for (uint32_t q = 0; q < n; ++q) {
        if ((la[q] >> 1) >= c->N() || (lb[q] >> 1) >= c->N() || cut_off[q + 1] < cut_off[q])
            return fail(c, CEC_E_ARG, "check %u: bad literal or cut offsets", q);
        std::vector<uint32_t> L(leaves + cut_off[q], leaves + cut_off[q + 1]);
        for (uint32_t x : L)
            if (x == 0 || x >= c->N()) return fail(c, CEC_E_ARG, "check %u: leaf out of range (or constant)", q);
        std::sort(L.begin(), L.end());  // increasing id (reading Q15)
        L.erase(std::unique(L.begin(), L.end()), L.end());
        if (L.size() > kcap) return fail(c, CEC_E_ARG, "check %u: %zu leaves > %u", q, L.size(), kcap);
        P->k[q] = (uint32_t)L.size();
        // cut validation: no PI outside L reachable from a root without crossing L.
        // Skipped for the Alg. 2 pass's own common cuts (trusted_cuts): u | v with u a cut of one root
        // and v of the other is a cut of both by construction (CEC_VALIDATE_CUTS=1 checks them anyway)
        bool ok = true;
        static const bool force_validate = getenv("CEC_VALIDATE_CUTS") != nullptr;
        if (!trusted_cuts || force_validate) {
            ++sep;
            for (uint32_t x : L) stop[x] = sep;
            uint32_t roots[2] = {la[q] >> 1, lb[q] >> 1};
            walk_tfi(c, c->scratch, roots, 2, &stop, sep, [&](uint32_t v) {
                if (v >= 1 && v <= c->I && stop[v] != sep) ok = false;
            });
        }
        if (!ok) {
            P->pre_verdict[q] = CEC_BAD_CUT;
            if (!bad++) first_bad = q;
            continue;
        }
        if (la[q] == lb[q]) {
            P->pre_verdict[q] = CEC_EQUIVALENT;
            continue;
        }
        if (la[q] == (lb[q] ^ 1u)) {
            P->pre_verdict[q] = CEC_UNDECIDED;
            continue;
        }
        P->pre_verdict[q] = DECIDED_BY_SIM;
        Cmp cm;
        cm.la = la[q];
        cm.lb = lb[q];
        cm.S = L;
        P->pair_cmp[q] = (int32_t)P->cmps.size();
        WinHost w;  // no merging for local checks
        w.inputs = L;
        w.cmps.push_back((uint32_t)P->cmps.size());
        P->cmps.push_back(std::move(cm));
        wins.push_back(std::move(w));
    }
    cec_status st = finish_plan(c, P.get(), wins, &stop, true);
    if (st != CEC_OK) return st;
    P->host_ms = std::chrono::duration<float, std::milli>(std::chrono::steady_clock::now() - t0).count();
    c->stats.host_prep_ms = P->host_ms;
    st = upload(c, P.get());
    if (st == CEC_OK && !P->cmps.empty()) st = cec_plan_run(c, P.get());
    if (st != CEC_OK) {
        free_dev(P.get());
        return st;
    }
    if (bad_out) *bad_out = bad;
    if (first_bad_out) *first_bad_out = first_bad;
    out = std::move(P);
    return CEC_OK;
}

cec_status local_checks_collect(cec_ctx *c, cec_plan *P, int32_t *verdict) {
    cec_status st = cec_plan_results(c, P, verdict, nullptr, nullptr);
    free_dev(P);
    return st;
}
