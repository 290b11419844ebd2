// supp_gpu.cu — a2 structural supports on the device (PAPER.md:23 "support", :81 window inputs).
//
// supp(PI) = {PI}, supp(const0) = {}, supp(AND n) = supp(f0) U supp(f1), as sorted PI-id lists
// saturating at `cap` = min(k_max, 41) + 1 <= 42 entries (a list of cap entries means "more than
// k_max": the pair is routed away from exhaustive simulation, and the host recomputes its exact k
// by a cone walk). One launch per topological level (cec_ensure_device_aig's CSR), one warp per
// node; then one warp per pair merges the two root lists (C5: 247 levels, 1.8 ms in total). The node lists live in one
// device block of N x cap u32 (C5: 2M nodes x 33 = 270 MB) that is a property of the AIG: it is built
// on a context's first call and kept; every call runs only the per-pair merge.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <vector>

#include "cec_internal.hpp"

namespace cec {
namespace {

__global__ void supp_init(uint32_t *lists, uint32_t *cnt, uint32_t I, uint32_t cap) {
    const uint32_t id = blockIdx.x * blockDim.x + threadIdx.x;
    if (id > I) return;
    cnt[id] = id ? 1u : 0u;
    lists[(size_t)id * cap] = id;
}

// One warp per node: both fanin lists are staged in shared memory (one coalesced load each) and
// every element's output rank comes from a binary search in the other list:
// rank(x in A) = i + lb(B, x) - #{dup b < x},  rank(y in B, not in A) = lb(A, y) + j - #{dup b < y}
__device__ __forceinline__ uint32_t lower_bound_s(const uint32_t *s, uint32_t n, uint32_t v) {
    uint32_t lo = 0, hi = n;
    while (lo < hi) {
        const uint32_t mid = (lo + hi) >> 1;
        if (s[mid] < v) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}
__device__ __forceinline__ uint32_t warp_union_smem(const uint32_t *__restrict__ A, uint32_t na,
                                                    const uint32_t *__restrict__ B, uint32_t nb, uint32_t *__restrict__ out,
                                                    uint32_t cap, uint32_t lane, uint32_t *sa, uint32_t *sb) {
    if (lane < na) sa[lane] = A[lane];
    if (lane + 32 < na) sa[lane + 32] = A[lane + 32];
    if (lane < nb) sb[lane] = B[lane];
    if (lane + 32 < nb) sb[lane + 32] = B[lane + 32];
    __syncwarp();
    bool d0 = false, d1 = false;
    uint32_t y0 = 0, y1 = 0, la0 = 0, la1 = 0;
    if (lane < nb) {
        y0 = sb[lane];
        la0 = lower_bound_s(sa, na, y0);
        d0 = la0 < na && sa[la0] == y0;
    }
    if (lane + 32 < nb) {
        y1 = sb[lane + 32];
        la1 = lower_bound_s(sa, na, y1);
        d1 = la1 < na && sa[la1] == y1;
    }
    const unsigned long long dm =
        (unsigned long long)__ballot_sync(0xFFFFFFFFu, d0) | ((unsigned long long)__ballot_sync(0xFFFFFFFFu, d1) << 32);
    const uint32_t total = na + nb - (uint32_t)__popcll(dm);
    auto dups_below = [&](uint32_t pos) {  // duplicate b elements at positions < pos
        return (uint32_t)__popcll(pos >= 64 ? dm : (dm & ((1ull << pos) - 1ull)));
    };
    for (uint32_t i = lane; i < na; i += 32) {
        const uint32_t x = sa[i], lb = lower_bound_s(sb, nb, x);
        const uint32_t r = i + lb - dups_below(lb);
        if (r < cap) out[r] = x;
    }
    if (lane < nb && !d0) {
        const uint32_t r = la0 + lane - dups_below(lane);
        if (r < cap) out[r] = y0;
    }
    if (lane + 32 < nb && !d1) {
        const uint32_t r = la1 + lane + 32 - dups_below(lane + 32);
        if (r < cap) out[r] = y1;
    }
    __syncwarp();
    return total < cap ? total : cap;
}

__global__ void supp_level_smem(const uint32_t *__restrict__ ids, uint32_t n, const uint32_t *__restrict__ f0,
                                const uint32_t *__restrict__ f1, uint32_t *lists, uint32_t *cnt, uint32_t cap) {
    __shared__ uint32_t sh[8][128];
    const uint32_t lane = threadIdx.x & 31u, wib = threadIdx.x >> 5;
    const uint32_t nw = gridDim.x * blockDim.x / 32;
    for (uint32_t t = (blockIdx.x * blockDim.x + threadIdx.x) / 32; t < n; t += nw) {
        const uint32_t id = ids[t], a = f0[id] >> 1, b = f1[id] >> 1;
        const uint32_t na = cnt[a], nb = cnt[b];
        uint32_t r = cap;
        if (na < cap && nb < cap)
            r = warp_union_smem(lists + (size_t)a * cap, na, lists + (size_t)b * cap, nb, lists + (size_t)id * cap, cap,
                                lane, sh[wib], sh[wib] + 64);
        if (lane == 0) cnt[id] = r;
    }
}

// one warp per pair: union of the two root lists
__global__ void supp_pairs(const uint2 *__restrict__ roots, uint32_t n, const uint32_t *__restrict__ lists,
                           const uint32_t *__restrict__ cnt, uint32_t cap, uint32_t *out, uint32_t *out_cnt) {
    __shared__ uint32_t sh[8][128];
    const uint32_t lane = threadIdx.x & 31u, wib = threadIdx.x >> 5;
    const uint32_t nw = gridDim.x * blockDim.x / 32;
    for (uint32_t p = (blockIdx.x * blockDim.x + threadIdx.x) / 32; p < n; p += nw) {
        const uint2 r = roots[p];
        const uint32_t na = cnt[r.x], nb = cnt[r.y];
        uint32_t c = cap;
        if (na < cap && nb < cap)
            c = warp_union_smem(lists + (size_t)r.x * cap, na, lists + (size_t)r.y * cap, nb, out + (size_t)p * cap, cap, lane,
                                sh[wib], sh[wib] + 64);
        if (lane == 0) out_cnt[p] = c;
    }
}

inline const char *ck(cudaError_t e) { return e == cudaSuccess ? nullptr : cudaGetErrorString(e); }

// Cone sizes for the cost-aware merge: |TFI(a) u TFI(b)| in AND nodes (roots included, PIs and the
// constant excluded), one block per pair: a breadth-first walk whose visited set is an
// open-addressing hash table in shared memory and whose frontiers are two shared arrays. A cone that
// does not fit (hash over half full, frontier overflow) reports UINT32_MAX and is walked on the host.
constexpr uint32_t CONE_HS = 8192, CONE_FC = 4096, CONE_EMPTY = 0xFFFFFFFFu;
constexpr size_t CONE_SMEM = sizeof(uint32_t) * (CONE_HS + 2 * CONE_FC);

__device__ __forceinline__ int cone_insert(uint32_t *keys, uint32_t key) {  // 1 new, 0 present, -1 full
    uint32_t h = (key * 0x9E3779B1u) >> (32 - 13);  // 13 = log2(CONE_HS)
    for (uint32_t probe = 0; probe < 64; ++probe) {
        const uint32_t old = atomicCAS(&keys[h], CONE_EMPTY, key);
        if (old == CONE_EMPTY) return 1;
        if (old == key) return 0;
        h = (h + 1) & (CONE_HS - 1);
    }
    return -1;
}

__global__ void __launch_bounds__(256) cone_sizes(const uint2 *__restrict__ roots, uint32_t n,
                                                  const uint32_t *__restrict__ f0, const uint32_t *__restrict__ f1,
                                                  uint32_t I, uint32_t *out) {
    extern __shared__ uint32_t sm[];
    uint32_t *keys = sm, *fr[2] = {sm + CONE_HS, sm + CONE_HS + CONE_FC};
    __shared__ uint32_t s_cnt, s_nf[2], s_over;
    for (uint32_t p = blockIdx.x; p < n; p += gridDim.x) {
        for (uint32_t i = threadIdx.x; i < CONE_HS; i += blockDim.x) keys[i] = CONE_EMPTY;
        if (threadIdx.x == 0) s_cnt = 0, s_nf[0] = 0, s_nf[1] = 0, s_over = 0;
        __syncthreads();
        if (threadIdx.x < 2) {
            const uint32_t r = threadIdx.x ? roots[p].y : roots[p].x;
            if (r > I) {
                const int ins = cone_insert(keys, r);
                if (ins < 0) s_over = 1;
                if (ins > 0) {
                    atomicAdd(&s_cnt, 1u);
                    fr[0][atomicAdd(&s_nf[0], 1u)] = r;
                }
            }
        }
        __syncthreads();
        for (uint32_t cur = 0;; cur ^= 1u) {
            const uint32_t nf = s_nf[cur];
            if (nf == 0 || s_over) break;
            if (threadIdx.x == 0) s_nf[cur ^ 1u] = 0;
            __syncthreads();
            for (uint32_t i = threadIdx.x; i < nf; i += blockDim.x) {
                const uint32_t v = fr[cur][i];
                const uint32_t fa[2] = {f0[v] >> 1, f1[v] >> 1};
                for (int t = 0; t < 2; ++t) {
                    if (fa[t] <= I) continue;  // PI or constant: not part of the AND cone
                    const int ins = cone_insert(keys, fa[t]);
                    if (ins < 0) s_over = 1;
                    if (ins <= 0) continue;
                    atomicAdd(&s_cnt, 1u);
                    const uint32_t slot = atomicAdd(&s_nf[cur ^ 1u], 1u);
                    if (slot < CONE_FC) fr[cur ^ 1u][slot] = fa[t];
                    else s_over = 1;
                }
            }
            __syncthreads();
        }
        if (threadIdx.x == 0) out[p] = (s_over || s_cnt > CONE_HS / 2) ? 0xFFFFFFFFu : s_cnt;
        __syncthreads();
    }
}

}  // namespace

const char *gpu_cones(DevPool &pool, const uint32_t *d_f0, const uint32_t *d_f1, uint32_t I,
                      const std::vector<uint2> &roots, std::vector<uint32_t> &cone_out, void *stream) {
    cudaStream_t st = (cudaStream_t)stream;
    const uint32_t n = (uint32_t)roots.size();
    cone_out.assign(n, 0xFFFFFFFFu);
    if (!n) return nullptr;
    auto al = [](size_t x) { return (x + 255) / 256 * 256; };
    const size_t b_roots = al(sizeof(uint2) * n), b_out = al(sizeof(uint32_t) * n);
    void *blk = nullptr;
    size_t blk_cap = 0;
    const char *e;
    if ((e = pool.get(b_roots + b_out, &blk, &blk_cap))) return e;
    uint2 *d_roots = (uint2 *)blk;
    uint32_t *d_out = (uint32_t *)((char *)blk + b_roots);
    if ((e = ck(cudaFuncSetAttribute(cone_sizes, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)CONE_SMEM)))) {
        pool.put(blk, blk_cap);
        return e;
    }
    e = ck(cudaMemcpyAsync(d_roots, roots.data(), sizeof(uint2) * n, cudaMemcpyHostToDevice, st));
    if (!e) {
        cone_sizes<<<(unsigned)std::min<uint32_t>(n, 148u * 3u), 256, CONE_SMEM, st>>>(d_roots, n, d_f0, d_f1, I, d_out);
        e = ck(cudaGetLastError());
    }
    if (!e) e = ck(cudaMemcpyAsync(cone_out.data(), d_out, sizeof(uint32_t) * n, cudaMemcpyDeviceToHost, st));
    if (!e) e = ck(cudaStreamSynchronize(st));
    if (e) cudaStreamSynchronize(st);
    pool.put(blk, blk_cap);
    return e;
}

const char *gpu_supports(DevPool &pool, const uint32_t *d_f0, const uint32_t *d_f1, const uint32_t *d_level_ids,
                         const std::vector<uint32_t> &level_off, uint32_t I, uint32_t N, uint32_t cap,
                         const std::vector<uint2> &roots, std::vector<uint32_t> &lists_out,
                         std::vector<uint32_t> &cnt_out, void *stream, uint32_t *launches, NodeSupports *table) {
    cudaStream_t st = (cudaStream_t)stream;
    const uint32_t n = (uint32_t)roots.size();
    auto al = [](size_t x) { return (x + 255) / 256 * 256; };
    const size_t b_roots = al(sizeof(uint2) * std::max<uint32_t>(n, 1)),
                 b_out = al(sizeof(uint32_t) * (size_t)std::max<uint32_t>(n, 1) * cap),
                 b_ocnt = al(sizeof(uint32_t) * std::max<uint32_t>(n, 1));
    void *blk = nullptr;
    size_t blk_cap = 0;
    const char *e;
    if (cap > 64) return "support cap above 64";
    if ((e = pool.get(b_roots + b_out + b_ocnt, &blk, &blk_cap))) return e;
    char *base = (char *)blk;
    uint2 *d_roots = (uint2 *)base;
    uint32_t *out = (uint32_t *)(base + b_roots), *ocnt = (uint32_t *)(base + b_roots + b_out);
    uint32_t nl = 0;
    const int T = 256;
    auto fail = [&](const char *m) {
        cudaStreamSynchronize(st);
        pool.put(blk, blk_cap);
        return m;
    };
    if ((e = ck(cudaMemcpyAsync(d_roots, roots.data(), sizeof(uint2) * n, cudaMemcpyHostToDevice, st)))) return fail(e);
    auto wgrid = [&](uint32_t m) { return (unsigned)std::min<uint64_t>(148ull * 16, ((uint64_t)m * 32 + T - 1) / T); };
    // The per-node table depends on the AIG only (like its levels, a1): built on the context's first
    // call, kept in device memory and reused by every later call with the same cap.
    if (!table->lists || table->cap != cap) {
        if (table->lists) cudaFree(table->lists);
        table->lists = nullptr;
        table->cnt = nullptr;
        void *tb = nullptr;
        const size_t b_lists = al(sizeof(uint32_t) * (size_t)N * cap), b_cnt = al(sizeof(uint32_t) * N);
        if ((e = ck(cudaMalloc(&tb, b_lists + b_cnt)))) return fail(e);
        table->lists = (uint32_t *)tb;
        table->cnt = (uint32_t *)((char *)tb + b_lists);
        table->cap = cap;
        supp_init<<<(I + 1 + T - 1) / T, T, 0, st>>>(table->lists, table->cnt, I, cap);
        ++nl;
        for (size_t l = 1; l + 1 < level_off.size(); ++l) {  // one launch per topological level
            const uint32_t b = level_off[l], m = level_off[l + 1] - b;
            if (!m) continue;
            supp_level_smem<<<wgrid(m), T, 0, st>>>(d_level_ids + b, m, d_f0, d_f1, table->lists, table->cnt, cap);
            ++nl;
        }
        table->launches = nl;
    }
    uint32_t *lists = table->lists, *cnt = table->cnt;
    if (n) {
        supp_pairs<<<wgrid(n), T, 0, st>>>(d_roots, n, lists, cnt, cap, out, ocnt);
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
