// supp_gpu.cu — a2 structural supports on the device (PAPER.md:23 "support", :81 window inputs).
//
// supp(PI) = {PI}, supp(const0) = {}, supp(AND n) = supp(f0) U supp(f1), as sorted PI-id lists
// saturating at `cap` = k_max + 1 entries (a list of cap entries means "more than k_max": the pair
// is routed away from exhaustive simulation, and the host recomputes its exact k by a cone walk).
// One launch per topological level, one thread per node (the level CSR of cec_ensure_device_aig);
// then one thread per pair merges the two root lists. Lists live in one device block of
// N x cap u32 (C5: 2M nodes x 33 = 270 MB, written once and read twice per call: ~0.3 ms of HBM).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <vector>

#include "cec_internal.hpp"

namespace cec {
namespace {

__device__ __forceinline__ uint32_t merge_capped(const uint32_t *__restrict__ a, uint32_t na,
                                                 const uint32_t *__restrict__ b, uint32_t nb, uint32_t *__restrict__ out,
                                                 uint32_t cap) {
    uint32_t i = 0, j = 0, n = 0;
    while (n < cap && (i < na || j < nb)) {
        uint32_t v;
        if (j >= nb || (i < na && a[i] < b[j])) {
            v = a[i++];
        } else if (i >= na || b[j] < a[i]) {
            v = b[j++];
        } else {
            v = a[i++];
            ++j;
        }
        out[n++] = v;
    }
    return n;
}

__global__ void supp_init(uint32_t *lists, uint32_t *cnt, uint32_t I, uint32_t cap) {
    const uint32_t id = blockIdx.x * blockDim.x + threadIdx.x;
    if (id > I) return;
    cnt[id] = id ? 1u : 0u;
    lists[(size_t)id * cap] = id;
}

__global__ void supp_level(const uint32_t *__restrict__ ids, uint32_t n, const uint32_t *__restrict__ f0,
                           const uint32_t *__restrict__ f1, uint32_t *lists, uint32_t *cnt, uint32_t cap) {
    const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= n) return;
    const uint32_t id = ids[t], a = f0[id] >> 1, b = f1[id] >> 1;
    const uint32_t na = cnt[a], nb = cnt[b];
    cnt[id] = (na >= cap || nb >= cap) ? cap
                                       : merge_capped(lists + (size_t)a * cap, na, lists + (size_t)b * cap, nb,
                                                      lists + (size_t)id * cap, cap);
}

__global__ void supp_pairs(const uint2 *__restrict__ roots, uint32_t n, const uint32_t *__restrict__ lists,
                           const uint32_t *__restrict__ cnt, uint32_t cap, uint32_t *out, uint32_t *out_cnt) {
    const uint32_t p = blockIdx.x * blockDim.x + threadIdx.x;
    if (p >= n) return;
    const uint2 r = roots[p];
    const uint32_t na = cnt[r.x], nb = cnt[r.y];
    out_cnt[p] = (na >= cap || nb >= cap)
                     ? cap
                     : merge_capped(lists + (size_t)r.x * cap, na, lists + (size_t)r.y * cap, nb, out + (size_t)p * cap, cap);
}

inline const char *ck(cudaError_t e) { return e == cudaSuccess ? nullptr : cudaGetErrorString(e); }

}  // namespace

const char *gpu_supports(DevPool &pool, const uint32_t *d_f0, const uint32_t *d_f1, const uint32_t *d_level_ids,
                         const std::vector<uint32_t> &level_off, uint32_t I, uint32_t N, uint32_t cap,
                         const std::vector<uint2> &roots, std::vector<uint32_t> &lists_out,
                         std::vector<uint32_t> &cnt_out, void *stream, uint32_t *launches) {
    cudaStream_t st = (cudaStream_t)stream;
    const uint32_t n = (uint32_t)roots.size();
    auto al = [](size_t x) { return (x + 255) / 256 * 256; };
    const size_t b_lists = al(sizeof(uint32_t) * (size_t)N * cap), b_cnt = al(sizeof(uint32_t) * N),
                 b_roots = al(sizeof(uint2) * std::max<uint32_t>(n, 1)),
                 b_out = al(sizeof(uint32_t) * (size_t)std::max<uint32_t>(n, 1) * cap),
                 b_ocnt = al(sizeof(uint32_t) * std::max<uint32_t>(n, 1));
    void *blk = nullptr;
    size_t blk_cap = 0;
    const char *e;
    if ((e = pool.get(b_lists + b_cnt + b_roots + b_out + b_ocnt, &blk, &blk_cap))) return e;
    char *base = (char *)blk;
    uint32_t *lists = (uint32_t *)base, *cnt = (uint32_t *)(base + b_lists);
    uint2 *d_roots = (uint2 *)(base + b_lists + b_cnt);
    uint32_t *out = (uint32_t *)(base + b_lists + b_cnt + b_roots), *ocnt = (uint32_t *)(base + b_lists + b_cnt + b_roots + b_out);
    uint32_t nl = 0;
    const int T = 256;
    auto fail = [&](const char *m) {
        cudaStreamSynchronize(st);
        pool.put(blk, blk_cap);
        return m;
    };
    if ((e = ck(cudaMemcpyAsync(d_roots, roots.data(), sizeof(uint2) * n, cudaMemcpyHostToDevice, st)))) return fail(e);
    supp_init<<<(I + 1 + T - 1) / T, T, 0, st>>>(lists, cnt, I, cap);
    ++nl;
    for (size_t l = 1; l + 1 < level_off.size(); ++l) {
        const uint32_t b = level_off[l], m = level_off[l + 1] - b;
        if (!m) continue;
        supp_level<<<(m + T - 1) / T, T, 0, st>>>(d_level_ids + b, m, d_f0, d_f1, lists, cnt, cap);
        ++nl;
    }
    if (n) {
        supp_pairs<<<(n + T - 1) / T, T, 0, st>>>(d_roots, n, lists, cnt, cap, out, ocnt);
        ++nl;
    }
    if ((e = ck(cudaGetLastError()))) return fail(e);
    lists_out.resize((size_t)n * cap);
    cnt_out.resize(n);
    if (n) {
        if ((e = ck(cudaMemcpyAsync(lists_out.data(), out, sizeof(uint32_t) * (size_t)n * cap, cudaMemcpyDeviceToHost, st))))
            return fail(e);
        if ((e = ck(cudaMemcpyAsync(cnt_out.data(), ocnt, sizeof(uint32_t) * n, cudaMemcpyDeviceToHost, st)))) return fail(e);
    }
    if ((e = ck(cudaStreamSynchronize(st)))) return fail(e);
    pool.put(blk, blk_cap);
    if (launches) *launches = nl;
    return nullptr;
}

}  // namespace cec
