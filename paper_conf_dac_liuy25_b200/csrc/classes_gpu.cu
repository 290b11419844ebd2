// classes_gpu.cu — equivalence classes from partial simulation, on the GPU (§II-B
// "nodes with identical partial truth tables are put into the same equivalence class", :61, :183,
// :187 CEX patterns split classes, kernels K4 + K5).
//
// Definition (oracle/classes.py, which shares no code with this file): every node is simulated on
// 32*(Wr + Wc) patterns — Wr random words per PI from the counter-based generator
// splitmix64(seed ^ (pi << 32) ^ w), then Wc caller words (e.g. counter-examples); nodes whose value
// vectors are equal or complementary form a class, representative = minimum id; every AND member
// yields (repr, member, relative phase), ordered by member id.
//
// GPU pipeline (all on the device, one D2H of the pairs at the end):
//   1. PI rows (random words generated in place, caller words copied), node-major table tt[id][W]
//      in HBM, one launch per level (random_sim, sim_random.cu), complement-canonical 64-bit
//      signature per node (canonical: pattern 0 evaluates to 0);
//   2. radix sort of (signature, id) — stable, so equal signatures keep ascending ids;
//   3. segment starts by a max-scan of head flags;
//   4. exactness: each node compares its canonical row with the rows before it in its segment and
//      takes the FIRST equal one as representative (= the class minimum id). A hash collision can
//      only put two classes in one segment; the row compare separates them, so the classes are
//      exactly the definition's, never a hash artefact;
//   5. flags -> exclusive scan -> pairs compacted in member-id order.
#include <cub/cub.cuh>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <vector>

#include "cec_internal.hpp"
#include "dev_util.cuh"

namespace cec {
namespace {

__device__ __forceinline__ uint64_t sm64(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}

__global__ void cl_pis(uint32_t *tt, uint32_t I, uint32_t W, uint32_t Wr, uint64_t seed, const uint32_t *__restrict__ cw,
                       uint32_t Wc) {
    const uint64_t n = (uint64_t)(I + 1) * W;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t id = i / W, w = i % W;
        uint32_t v = 0u;  // id 0 = constant 0
        if (id > 0) v = w < Wr ? (uint32_t)sm64(seed ^ (id << 32) ^ w) : cw[(id - 1) * Wc + (w - Wr)];
        tt[i] = v;
    }
}

__global__ void cl_iota(uint32_t *v, uint32_t n) {
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) v[i] = i;
}

__global__ void cl_heads(const unsigned long long *__restrict__ key, uint32_t n, uint32_t *head) {
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
        head[i] = (i == 0 || key[i] != key[i - 1]) ? i : 0u;
}

struct MaxU32 {
    __device__ __forceinline__ uint32_t operator()(uint32_t a, uint32_t b) const { return a > b ? a : b; }
};

__global__ void cl_find(const uint32_t *__restrict__ tt, uint32_t W, const uint32_t *__restrict__ ids,
                        const uint32_t *__restrict__ seg, const uint8_t *__restrict__ phase, uint32_t n, uint32_t I,
                        uint32_t *flag, uint32_t *rep, uint8_t *rph) {
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
        const uint32_t id = ids[i];
        const uint32_t inv = 0u - (uint32_t)phase[id];
        const uint32_t *row = tt + (uint64_t)id * W;
        uint32_t r = id;
        for (uint32_t j = seg[i]; j < i; ++j) {
            const uint32_t o = ids[j];
            const uint32_t oinv = 0u - (uint32_t)phase[o];
            const uint32_t *orow = tt + (uint64_t)o * W;
            bool eq = true;
            for (uint32_t w = 0; w < W && eq; ++w) eq = ((row[w] ^ inv) == (orow[w] ^ oinv));
            if (eq) {
                r = o;
                break;
            }
        }
        const bool member = r != id && id > I;
        flag[id] = member ? 1u : 0u;
        rep[id] = r;
        rph[id] = (uint8_t)(phase[id] ^ phase[r]);
    }
}

__global__ void cl_scatter(const uint32_t *__restrict__ flag, const uint32_t *__restrict__ pos,
                           const uint32_t *__restrict__ rep, const uint8_t *__restrict__ rph, uint32_t N, uint32_t cap,
                           uint32_t *out_r, uint32_t *out_m, uint8_t *out_p) {
    for (uint32_t id = blockIdx.x * blockDim.x + threadIdx.x; id < N; id += gridDim.x * blockDim.x)
        if (flag[id] && pos[id] < cap) {
            out_r[pos[id]] = rep[id];
            out_m[pos[id]] = id;
            out_p[pos[id]] = rph[id];
        }
}

inline const char *ck(cudaError_t e) { return e == cudaSuccess ? nullptr : cudaGetErrorString(e); }

}  // namespace

const char *gpu_classes(const uint32_t *d_f0, const uint32_t *d_f1, const uint32_t *d_level_ids,
                        const std::vector<uint32_t> &level_off, uint32_t I, uint32_t N, uint32_t Wr, uint64_t seed,
                        uint32_t Wc, const uint32_t *h_words, uint32_t cap, void *stream, int num_sms,
                        DevPool *pool, uint32_t *total_out, std::vector<uint32_t> &repr,
                        std::vector<uint32_t> &member, std::vector<uint8_t> &phase, uint32_t *launches,
                        float *kernel_ms) {
    cudaStream_t st = (cudaStream_t)stream;
    const uint32_t W = Wr + Wc;
    size_t sort_bytes = 0, scan_bytes = 0, mscan_bytes = 0;
    cub::DeviceRadixSort::SortPairs(nullptr, sort_bytes, (const unsigned long long *)nullptr,
                                    (unsigned long long *)nullptr, (const uint32_t *)nullptr, (uint32_t *)nullptr, (int)N,
                                    0, 64, st);
    cub::DeviceScan::ExclusiveSum(nullptr, scan_bytes, (uint32_t *)nullptr, (uint32_t *)nullptr, (int)N, st);
    cub::DeviceScan::InclusiveScan(nullptr, mscan_bytes, (uint32_t *)nullptr, (uint32_t *)nullptr, MaxU32(), (int)N, st);
    const size_t tmp_bytes = std::max(sort_bytes, std::max(scan_bytes, mscan_bytes));
    const uint32_t ocap = std::max<uint32_t>(cap, 1);
    // layout (256-B aligned pieces)
    size_t off = 0;
    auto take = [&](size_t b) {
        const size_t o = off;
        off += (b + 255) & ~(size_t)255;
        return o;
    };
    const size_t o_tt = take(4ull * N * W), o_sig = take(8ull * N), o_sig2 = take(8ull * N), o_ph = take(N),
                 o_ids = take(4ull * N), o_ids2 = take(4ull * N), o_seg = take(4ull * N), o_flag = take(4ull * N),
                 o_pos = take(4ull * N), o_rep = take(4ull * N), o_rph = take(N), o_cw = take(4ull * I * Wc + 4),
                 o_or = take(4ull * ocap), o_om = take(4ull * ocap), o_op = take(ocap), o_tmp = take(tmp_bytes);
    const char *e;
    DevBlock B{pool, st};
    if ((e = B.alloc(off))) return e;
    char *blk = (char *)B.p;
    EventPair ev;
    if ((e = ev.create())) return e;
    uint32_t *tt = (uint32_t *)(blk + o_tt), *ids = (uint32_t *)(blk + o_ids), *ids2 = (uint32_t *)(blk + o_ids2);
    unsigned long long *sig = (unsigned long long *)(blk + o_sig), *sig2 = (unsigned long long *)(blk + o_sig2);
    uint8_t *ph = (uint8_t *)(blk + o_ph), *rph = (uint8_t *)(blk + o_rph), *op = (uint8_t *)(blk + o_op);
    uint32_t *seg = (uint32_t *)(blk + o_seg), *flag = (uint32_t *)(blk + o_flag), *pos = (uint32_t *)(blk + o_pos);
    uint32_t *rep = (uint32_t *)(blk + o_rep), *cw = (uint32_t *)(blk + o_cw), *orr = (uint32_t *)(blk + o_or),
             *om = (uint32_t *)(blk + o_om);
    void *tmp = blk + o_tmp;
    const int T = 256;
    const unsigned gcap = (unsigned)std::max(1, num_sms * 8);
    auto grid = [&](uint64_t work) { return (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(gcap, (work + T - 1) / T)); };
    uint32_t nl = 0;
    if (Wc && (e = ck(cudaMemcpyAsync(cw, h_words, 4ull * I * Wc, cudaMemcpyHostToDevice, st)))) return e;
    if ((e = ck(cudaEventRecord(ev.a, st)))) return e;
    cl_pis<<<grid((uint64_t)(I + 1) * W), T, 0, st>>>(tt, I, W, Wr, seed, cw, Wc);
    ++nl;
    uint32_t nsim = 0;
    if ((e = random_sim(d_f0, d_f1, d_level_ids, level_off, I, N, W, seed, tt, sig, ph, stream, num_sms, &nsim, true)))
        return e;
    nl += nsim;
    cl_iota<<<grid(N), T, 0, st>>>(ids, N);
    ++nl;
    size_t tb = tmp_bytes;
    if ((e = ck(cub::DeviceRadixSort::SortPairs(tmp, tb, sig, sig2, ids, ids2, (int)N, 0, 64, st)))) return e;
    cl_heads<<<grid(N), T, 0, st>>>(sig2, N, seg);
    tb = tmp_bytes;
    if ((e = ck(cub::DeviceScan::InclusiveScan(tmp, tb, seg, pos, MaxU32(), (int)N, st)))) return e;  // pos = seg start
    cl_find<<<grid(N), T, 0, st>>>(tt, W, ids2, pos, ph, N, I, flag, rep, rph);
    tb = tmp_bytes;
    if ((e = ck(cub::DeviceScan::ExclusiveSum(tmp, tb, flag, pos, (int)N, st)))) return e;
    cl_scatter<<<grid(N), T, 0, st>>>(flag, pos, rep, rph, N, cap, orr, om, op);
    nl += 6;
    if ((e = ck(cudaGetLastError()))) return e;
    if ((e = ck(cudaEventRecord(ev.b, st)))) return e;
    uint32_t tail[2] = {0, 0};
    if ((e = ck(cudaMemcpyAsync(&tail[0], pos + (N - 1), 4, cudaMemcpyDeviceToHost, st)))) return e;
    if ((e = ck(cudaMemcpyAsync(&tail[1], flag + (N - 1), 4, cudaMemcpyDeviceToHost, st)))) return e;
    if ((e = ck(cudaStreamSynchronize(st)))) return e;
    const uint32_t total = tail[0] + tail[1], n = std::min(total, cap);
    repr.resize(n);
    member.resize(n);
    phase.resize(n);
    if (n) {
        if ((e = ck(cudaMemcpyAsync(repr.data(), orr, 4ull * n, cudaMemcpyDeviceToHost, st)))) return e;
        if ((e = ck(cudaMemcpyAsync(member.data(), om, 4ull * n, cudaMemcpyDeviceToHost, st)))) return e;
        if ((e = ck(cudaMemcpyAsync(phase.data(), op, n, cudaMemcpyDeviceToHost, st)))) return e;
        if ((e = ck(cudaStreamSynchronize(st)))) return e;
    }
    *total_out = total;
    if (launches) *launches = nl;
    if (kernel_ms) cudaEventElapsedTime(kernel_ms, ev.a, ev.b);
    return nullptr;
}

}  // namespace cec
