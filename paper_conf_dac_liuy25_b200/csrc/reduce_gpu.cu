// reduce_gpu.cu — miter reduction on the GPU ("the miter manager ... reduces the miter by
// merging the proved equivalent pairs", :185, :187, kernel K9).
//
// Definition (the same as oracle/reduce.py, which shares no code with this file): every AND in
// increasing id is either a proved member — its image is its representative's image (fanout
// redirection, representative = lower id) — or it is rebuilt from its fanins' images with
// the structural rules of an AIG package (x&0 = 0, x&1 = x, x&x = x, x&!x = 0) and hash-consing; new
// ids follow creation order (= increasing old id of the first node with that key).
//
// GPU formulation. Node images are computed batch by batch in a host-computed topological
// schedule (batch(n) > batch of every fanin, and > batch(repr) for a member), one thread per node.
// A rebuilt node is hash-consed in a device table keyed by its normalised fanin pair; its image is
// the table SLOT (label I+1+slot), not a node id, so every node with the same key gets the same
// label no matter which batch inserted the key first. atomicMin over the inserting old ids gives
// each slot the id the sequential definition would create it at (the first in id order). After
// the last batch, survivors (slot minima) are ranked by old id with one exclusive scan; a slot's
// new id is I+1+rank. That order is topological, and it is exactly the creation order of the
// sequential definition, so the output is identical to oracle/reduce.py, array for array.
//
// Memory: f0/f1 (the context's device AIG), sub[N], batch ids[N], lab[N], a 2x-oversized slot
// table (8 B key + 4 B id per slot), rank[N]. HBM-bound gathers; tiny next to the exhaustive sweep.
#include <cub/cub.cuh>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <vector>

#include "cec_internal.hpp"
#include "dev_util.cuh"

namespace cec {
namespace {

constexpr unsigned long long EMPTY_KEY = ~0ull;
constexpr uint32_t NONE = 0xFFFFFFFFu;

__device__ __forceinline__ uint32_t slot_hash(unsigned long long k) {
    k ^= k >> 33;
    k *= 0xFF51AFD7ED558CCDull;
    k ^= k >> 33;
    k *= 0xC4CEB9FE1A85EC53ull;
    k ^= k >> 33;
    return (uint32_t)k;
}

__global__ void rd_init(unsigned long long *keys, uint32_t *minid, uint32_t cap, uint32_t *lab, uint32_t I) {
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < cap; i += gridDim.x * blockDim.x) {
        keys[i] = EMPTY_KEY;
        minid[i] = NONE;
    }
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i <= I; i += gridDim.x * blockDim.x) lab[i] = 2u * i;
}

// One batch of the schedule: image label-literal of every node in ids[0..n).
__global__ void rd_batch(const uint32_t *__restrict__ ids, uint32_t n, const uint32_t *__restrict__ f0,
                         const uint32_t *__restrict__ f1, const uint32_t *__restrict__ sub, uint32_t *lab,
                         unsigned long long *keys, uint32_t *minid, uint32_t mask, uint32_t I, uint32_t *overflow) {
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    const uint32_t id = ids[i];
    const uint32_t s = sub[id];
    if (s != NONE) {  // proved member: redirect to the representative's image
        lab[id] = lab[s >> 1] ^ (s & 1u);
        return;
    }
    uint32_t a = lab[f0[id] >> 1] ^ (f0[id] & 1u), b = lab[f1[id] >> 1] ^ (f1[id] & 1u);
    if (a > b) {
        const uint32_t t = a;
        a = b;
        b = t;
    }
    uint32_t out;
    if (a == 0u || a == (b ^ 1u)) {
        out = 0u;
    } else if (a == 1u) {
        out = b;
    } else if (a == b) {
        out = a;
    } else {
        const unsigned long long key = ((unsigned long long)a << 32) | b;
        uint32_t h = slot_hash(key) & mask;
        for (uint32_t probe = 0;; ++probe) {
            const unsigned long long prev = atomicCAS(&keys[h], EMPTY_KEY, key);
            if (prev == EMPTY_KEY || prev == key) break;
            h = (h + 1u) & mask;
            if (probe > mask) {  // cannot happen with a 2x table; reported, never silent
                atomicExch(overflow, 1u);
                return;
            }
        }
        atomicMin(&minid[h], id);
        out = 2u * (I + 1u + h);
    }
    lab[id] = out;
}

__global__ void rd_flags(const uint32_t *__restrict__ minid, uint32_t cap, uint32_t *surv) {
    for (uint32_t h = blockIdx.x * blockDim.x + threadIdx.x; h < cap; h += gridDim.x * blockDim.x)
        if (minid[h] != NONE) surv[minid[h]] = 1u;
}

__device__ __forceinline__ uint32_t to_new(uint32_t lit, uint32_t I, const uint32_t *__restrict__ minid,
                                           const uint32_t *__restrict__ rank) {
    const uint32_t l = lit >> 1;
    if (l <= I) return lit;
    return 2u * (I + 1u + rank[minid[l - I - 1u]]) | (lit & 1u);
}

__global__ void rd_emit(const unsigned long long *__restrict__ keys, const uint32_t *__restrict__ minid, uint32_t cap,
                        const uint32_t *__restrict__ rank, uint32_t I, uint32_t *out_fanins) {
    for (uint32_t h = blockIdx.x * blockDim.x + threadIdx.x; h < cap; h += gridDim.x * blockDim.x) {
        if (minid[h] == NONE) continue;
        const uint32_t r = rank[minid[h]];
        uint32_t a = to_new((uint32_t)(keys[h] >> 32), I, minid, rank), b = to_new((uint32_t)keys[h], I, minid, rank);
        if (a > b) {
            const uint32_t t = a;
            a = b;
            b = t;
        }
        out_fanins[2u * r] = a;
        out_fanins[2u * r + 1u] = b;
    }
}

__global__ void rd_image(const uint32_t *__restrict__ lab, uint32_t N, uint32_t I, const uint32_t *__restrict__ minid,
                         const uint32_t *__restrict__ rank, uint32_t *image) {
    for (uint32_t id = blockIdx.x * blockDim.x + threadIdx.x; id < N; id += gridDim.x * blockDim.x)
        image[id] = to_new(lab[id], I, minid, rank);
}

inline const char *ck(cudaError_t e) { return e == cudaSuccess ? nullptr : cudaGetErrorString(e); }

}  // namespace

const char *gpu_reduce(const uint32_t *d_f0, const uint32_t *d_f1, uint32_t I, uint32_t N, const std::vector<uint32_t> &sub,
                       const std::vector<uint32_t> &batch_ids, const std::vector<uint32_t> &batch_off, void *stream,
                       int num_sms, DevPool *pool, std::vector<uint32_t> &new_fanins, std::vector<uint32_t> &image,
                       uint32_t *launches, float *kernel_ms) {
    cudaStream_t st = (cudaStream_t)stream;
    const uint32_t A = N - 1 - I;
    uint32_t cap = 1024;
    while (cap < 2u * std::max<uint32_t>(A, 1u)) cap <<= 1;
    // one device block: sub, ids, lab, surv, rank, img, minid [u32]; keys [u64]; overflow; scan temp
    size_t scan_bytes = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, scan_bytes, (uint32_t *)nullptr, (uint32_t *)nullptr, (int)N, st);
    const size_t n32 = 6 * (size_t)N + cap + 1 + 2 * (size_t)A + 4;
    const size_t bytes = 8 * (size_t)cap + 4 * n32 + scan_bytes + 256;
    const char *e;
    DevBlock B{pool, st};
    if ((e = B.alloc(bytes))) return e;
    char *blk = (char *)B.p;
    EventPair ev;
    if ((e = ev.create())) return e;
    unsigned long long *keys = (unsigned long long *)blk;
    uint32_t *p = (uint32_t *)(blk + 8 * (size_t)cap);
    uint32_t *d_sub = p, *d_ids = p + N, *lab = p + 2 * (size_t)N, *surv = p + 3 * (size_t)N, *rank = p + 4 * (size_t)N;
    uint32_t *img = p + 5 * (size_t)N, *minid = p + 6 * (size_t)N, *overflow = minid + cap, *out = overflow + 1;
    void *scan_tmp = (void *)(((uintptr_t)(out + 2 * (size_t)A + 3) + 255) & ~(uintptr_t)255);
    uint32_t nl = 0;
    if ((e = ck(cudaMemcpyAsync(d_sub, sub.data(), 4 * (size_t)N, cudaMemcpyHostToDevice, st)))) return e;
    if (!batch_ids.empty() &&
        (e = ck(cudaMemcpyAsync(d_ids, batch_ids.data(), 4 * batch_ids.size(), cudaMemcpyHostToDevice, st))))
        return e;
    if ((e = ck(cudaMemsetAsync(surv, 0, 4 * (size_t)N, st)))) return e;
    if ((e = ck(cudaMemsetAsync(overflow, 0, 4, st)))) return e;
    const int T = 256;
    const unsigned gcap = (unsigned)std::max(1, num_sms * 8);
    auto grid = [&](uint64_t work) { return (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(gcap, (work + T - 1) / T)); };
    if ((e = ck(cudaEventRecord(ev.a, st)))) return e;
    rd_init<<<grid(std::max<uint64_t>(cap, I + 1)), T, 0, st>>>(keys, minid, cap, lab, I);
    ++nl;
    for (size_t b = 0; b + 1 < batch_off.size(); ++b) {
        const uint32_t n = batch_off[b + 1] - batch_off[b];
        if (!n) continue;
        rd_batch<<<(n + T - 1) / T, T, 0, st>>>(d_ids + batch_off[b], n, d_f0, d_f1, d_sub, lab, keys, minid, cap - 1, I,
                                                overflow);
        ++nl;
    }
    if ((e = ck(cudaGetLastError()))) return e;
    rd_flags<<<grid(cap), T, 0, st>>>(minid, cap, surv);
    ++nl;
    if ((e = ck(cub::DeviceScan::ExclusiveSum(scan_tmp, scan_bytes, surv, rank, (int)N, st)))) return e;
    ++nl;
    rd_emit<<<grid(cap), T, 0, st>>>(keys, minid, cap, rank, I, out);
    rd_image<<<grid(N), T, 0, st>>>(lab, N, I, minid, rank, img);
    nl += 2;
    if ((e = ck(cudaGetLastError()))) return e;
    if ((e = ck(cudaEventRecord(ev.b, st)))) return e;
    uint32_t tail[2] = {0, 0}, ovf = 0;  // survivors = rank[N-1] + surv[N-1]
    if ((e = ck(cudaMemcpyAsync(&tail[0], rank + (N - 1), 4, cudaMemcpyDeviceToHost, st)))) return e;
    if ((e = ck(cudaMemcpyAsync(&tail[1], surv + (N - 1), 4, cudaMemcpyDeviceToHost, st)))) return e;
    if ((e = ck(cudaMemcpyAsync(&ovf, overflow, 4, cudaMemcpyDeviceToHost, st)))) return e;
    image.resize(N);
    if ((e = ck(cudaMemcpyAsync(image.data(), img, 4 * (size_t)N, cudaMemcpyDeviceToHost, st)))) return e;
    if ((e = ck(cudaStreamSynchronize(st)))) return e;
    if (ovf) return "reduction hash table overflow";
    const uint32_t Anew = tail[0] + tail[1];
    new_fanins.resize(2 * (size_t)Anew);
    if (Anew &&
        (e = ck(cudaMemcpyAsync(new_fanins.data(), out, 8 * (size_t)Anew, cudaMemcpyDeviceToHost, st))))
        return e;
    if ((e = ck(cudaStreamSynchronize(st)))) return e;
    if (launches) *launches = nl;
    if (kernel_ms) cudaEventElapsedTime(kernel_ms, ev.a, ev.b);
    return nullptr;
}

}  // namespace cec
