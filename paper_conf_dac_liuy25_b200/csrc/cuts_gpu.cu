// cuts_gpu.cu — GPU cut generator for local function checking (§III-C2, Alg. 2 :163-175;
// SURVEY.md §8(f) NEXT-1).
//
// Same definition as the host generator (csrc/cuts.cpp) and the cut oracle (oracle/cuts.py):
// Eq. (1) enumeration, dominated-cut removal, Table I ranking of the pass, similarity-guided
// ranking for non-representatives, lexicographic tie-break — bit-identical output.
// Parallel structure ("each cut in E(n) is generated using an individual thread, and the
// selection of the best C cuts ... jointly performed by the group of threads"):
//   * nodes are processed by enumeration level el(n) (Eq. 2): one launch per level, so a
//     representative's cuts exist before its members' (similarity) and fanins before fanouts;
//   * one warp per node: lanes generate the candidates u|v of E(n) (Eq. 1) into shared memory,
//     each lane decides for its candidates "dominated / duplicate" against all others, computes the
//     ranking keys, and ranks them by counting how many candidates precede them; the first C
//     are written as P(n);
//   * a second kernel forms the common cuts of each pair (one warp per pair) the same way.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <vector>

#include "cec_internal.hpp"

namespace cec {
namespace {

constexpr int KM = 24;            // max leaves (k_l <= 24)
constexpr int CMAX = 16;          // max priority cuts per node on the GPU
constexpr int EMAX = (CMAX + 1) * (CMAX + 1);
constexpr int WPB = 4;            // warps per block
constexpr uint32_t NONE = 0xFFFFFFFFu;

struct GCut {  // stored cut: n leaves, ascending
    uint32_t n;
    uint32_t leaf[KM];
};

struct Keys {
    unsigned long long sf, sl;  // sum of fanouts / levels of the leaves
    unsigned __int128 sim;      // similarity x lcm(1..48)
    uint32_t valid;
};

__device__ __forceinline__ bool dmerge(const uint32_t *a, uint32_t na, const uint32_t *b, uint32_t nb, uint32_t k,
                                       uint32_t *out, uint32_t &n) {
    uint32_t i = 0, j = 0;
    n = 0;
    while (i < na || j < nb) {
        uint32_t v;
        if (j >= nb || (i < na && a[i] < b[j])) {
            v = a[i++];
        } else if (i >= na || b[j] < a[i]) {
            v = b[j++];
        } else {
            v = a[i++];
            ++j;
        }
        if (n == k) return false;
        out[n++] = v;
    }
    return true;
}

__device__ __forceinline__ bool dsubset(const GCut &s, const GCut &b) {  // s ⊆ b
    if (s.n > b.n) return false;
    uint32_t j = 0;
    for (uint32_t i = 0; i < s.n; ++i) {
        while (j < b.n && b.leaf[j] < s.leaf[i]) ++j;
        if (j == b.n || b.leaf[j] != s.leaf[i]) return false;
        ++j;
    }
    return true;
}

__device__ __forceinline__ bool dequal(const GCut &a, const GCut &b) {
    if (a.n != b.n) return false;
    for (uint32_t i = 0; i < a.n; ++i)
        if (a.leaf[i] != b.leaf[i]) return false;
    return true;
}

__device__ __forceinline__ bool dlexless(const GCut &a, const GCut &b) {
    const uint32_t m = a.n < b.n ? a.n : b.n;
    for (uint32_t i = 0; i < m; ++i)
        if (a.leaf[i] != b.leaf[i]) return a.leaf[i] < b.leaf[i];
    return a.n < b.n;
}

__device__ __forceinline__ uint32_t dinter(const GCut &a, const GCut &b) {
    uint32_t i = 0, j = 0, c = 0;
    while (i < a.n && j < b.n) {
        if (a.leaf[i] == b.leaf[j]) {
            ++c;
            ++i;
            ++j;
        } else if (a.leaf[i] < b.leaf[j]) {
            ++i;
        } else {
            ++j;
        }
    }
    return c;
}

// strict total order of the pass (host cuts.cpp table1_less, with the similarity key first)
__device__ __forceinline__ bool rank_less(const GCut &a, const Keys &ka, const GCut &b, const Keys &kb, int pass,
                                          bool use_sim) {
    if (use_sim && ka.sim != kb.sim) return ka.sim > kb.sim;
    const unsigned long long fa = ka.sf * b.n, fb = kb.sf * a.n;
    const unsigned long long la = ka.sl * b.n, lb = kb.sl * a.n;
    if (pass == 0) {
        if (fa != fb) return fa > fb;
        if (a.n != b.n) return a.n < b.n;
        if (la != lb) return la < lb;
    } else if (pass == 1) {
        if (la != lb) return la < lb;
        if (a.n != b.n) return a.n < b.n;
        if (fa != fb) return fa > fb;
    } else {
        if (la != lb) return la > lb;
        if (a.n != b.n) return a.n < b.n;
        if (fa != fb) return fa > fb;
    }
    return dlexless(a, b);
}

__device__ unsigned __int128 d_lcm48() {
    unsigned __int128 l = 1;
    for (int i = 2; i <= 2 * KM; ++i) {
        unsigned __int128 a = l, b = (unsigned __int128)i;
        while (b) {
            unsigned __int128 t = a % b;
            a = b;
            b = t;
        }
        l = l / a * (unsigned __int128)i;
    }
    return l;
}

__device__ __forceinline__ void load_list(const GCut *P, const uint32_t *cnt, uint32_t C, uint32_t id, GCut *dst,
                                          uint32_t &n, uint32_t lane) {
    // P(id) followed by the trivial cut {id} (empty for the constant)
    const uint32_t c = cnt[id];
    for (uint32_t t = lane; t < c; t += 32) dst[t] = P[(size_t)id * C + t];
    if (lane == 0) {
        GCut &tr = dst[c];
        tr.n = id == 0 ? 0u : 1u;
        tr.leaf[0] = id;
    }
    n = c + 1;
}

__host__ __device__ constexpr size_t level_smem_per_warp() {
    return (sizeof(Keys) * EMAX + sizeof(GCut) * (2 * (CMAX + 1) + EMAX) + sizeof(uint32_t) * EMAX + 15) / 16 * 16;
}

__global__ void __launch_bounds__(WPB * 32)
cut_level_kernel(const uint32_t *__restrict__ nodes, uint32_t nnodes, const uint32_t *__restrict__ f0,
                 const uint32_t *__restrict__ f1, const uint32_t *__restrict__ fanout,
                 const uint32_t *__restrict__ level, const uint32_t *__restrict__ repr_of, GCut *P, uint32_t *cnt,
                 uint32_t k_l, uint32_t C, int pass) {
    extern __shared__ __align__(16) unsigned char sm[];
    const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31u;
    unsigned char *base = sm + level_smem_per_warp() * warp;
    Keys *K = reinterpret_cast<Keys *>(base);  // first: 16-byte aligned (__int128 member)
    GCut *Ua = reinterpret_cast<GCut *>(K + EMAX);
    GCut *Vb = Ua + (CMAX + 1);
    GCut *E = Vb + (CMAX + 1);
    uint32_t *rank = reinterpret_cast<uint32_t *>(E + EMAX);
    const unsigned __int128 L = d_lcm48();
    for (uint32_t w = blockIdx.x * WPB + warp; w < nnodes; w += gridDim.x * WPB) {
        const uint32_t id = nodes[w];
        const uint32_t a = f0[id] >> 1, b = f1[id] >> 1;
        uint32_t na, nb;
        load_list(P, cnt, C, a, Ua, na, lane);
        load_list(P, cnt, C, b, Vb, nb, lane);
        __syncwarp();
        const uint32_t ne = na * nb;
        for (uint32_t t = lane; t < ne; t += 32) {  // Eq. (1): one candidate per thread
            const GCut &u = Ua[t / nb], &v = Vb[t % nb];
            uint32_t n = 0;
            const bool ok = dmerge(u.leaf, u.n, v.leaf, v.n, k_l, E[t].leaf, n);
            E[t].n = n;
            K[t].valid = ok && n > 0 && !(n == 1 && E[t].leaf[0] == id);
        }
        __syncwarp();
        // dominated or duplicate (an equal candidate with a smaller index)
        for (uint32_t t = lane; t < ne; t += 32) {
            if (!K[t].valid) continue;
            bool drop = false;
            for (uint32_t o = 0; o < ne && !drop; ++o) {
                if (o == t || !K[o].valid) continue;
                if (E[o].n < E[t].n) drop = dsubset(E[o], E[t]);
                else if (E[o].n == E[t].n && o < t) drop = dequal(E[o], E[t]);
            }
            rank[t] = drop ? NONE : 0u;
        }
        __syncwarp();
        const uint32_t r = repr_of[id];
        const bool use_sim = r != NONE && cnt[r] > 0;
        for (uint32_t t = lane; t < ne; t += 32) {
            if (rank[t] == NONE || !K[t].valid) {
                K[t].valid = 0;
                continue;
            }
            unsigned long long sf = 0, sl = 0;
            for (uint32_t i = 0; i < E[t].n; ++i) {
                sf += fanout[E[t].leaf[i]];
                sl += level[E[t].leaf[i]];
            }
            K[t].sf = sf;
            K[t].sl = sl;
            unsigned __int128 s = 0;
            if (use_sim)
                for (uint32_t q = 0; q < cnt[r]; ++q) {
                    const GCut &y = P[(size_t)r * C + q];
                    const uint32_t in = dinter(E[t], y);
                    s += (unsigned __int128)in * (L / (unsigned __int128)(E[t].n + y.n - in));
                }
            K[t].sim = s;
        }
        __syncwarp();
        uint32_t kept = 0;
        for (uint32_t t = lane; t < ne; t += 32) {
            if (!K[t].valid) continue;
            uint32_t before = 0;
            for (uint32_t o = 0; o < ne; ++o)
                if (o != t && K[o].valid && rank_less(E[o], K[o], E[t], K[t], pass, use_sim)) ++before;
            if (before < C) P[(size_t)id * C + before] = E[t];
            ++kept;
        }
        for (int off = 16; off; off >>= 1) kept += __shfl_xor_sync(0xFFFFFFFFu, kept, off);
        if (lane == 0) cnt[id] = kept < C ? kept : C;
        __syncwarp();
    }
}

__global__ void __launch_bounds__(WPB * 32)
common_cut_kernel(const uint32_t *__restrict__ repr, const uint32_t *__restrict__ member, uint32_t npairs,
                  const GCut *__restrict__ P, const uint32_t *__restrict__ cnt, uint32_t k_l, uint32_t C,
                  uint32_t max_cuts, GCut *out, uint32_t *out_cnt) {
    extern __shared__ __align__(16) unsigned char sm[];
    const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31u;
    const size_t per_warp = sizeof(GCut) * (CMAX * CMAX) + sizeof(uint32_t) * (CMAX * CMAX);
    GCut *E = reinterpret_cast<GCut *>(sm + per_warp * warp);
    uint32_t *valid = reinterpret_cast<uint32_t *>(E + CMAX * CMAX);
    for (uint32_t q = blockIdx.x * WPB + warp; q < npairs; q += gridDim.x * WPB) {
        const uint32_t r = repr[q], m = member[q];
        const uint32_t nr = cnt[r], nm = cnt[m], ne = nr * nm;
        for (uint32_t t = lane; t < ne; t += 32) {
            const GCut &u = P[(size_t)r * C + t / nm], &v = P[(size_t)m * C + t % nm];
            uint32_t n = 0;
            const bool ok = dmerge(u.leaf, u.n, v.leaf, v.n, k_l, E[t].leaf, n);
            E[t].n = n;
            valid[t] = ok && n > 0;
        }
        __syncwarp();
        // drop duplicates (keep the smallest index) ...
        for (uint32_t t = lane; t < ne; t += 32) {
            bool v = valid[t];
            for (uint32_t o = 0; o < t && v; ++o)
                if (valid[o] && dequal(E[o], E[t])) v = false;
            valid[t] = v ? 2u : 0u;  // 2 = unique (written after every lane read the 0/1 flags)
        }
        __syncwarp();
        for (uint32_t t = lane; t < ne; t += 32) valid[t] = valid[t] == 2u;
        __syncwarp();
        // ... and order by (size, lexicographic)
        uint32_t kept = 0;
        for (uint32_t t = lane; t < ne; t += 32) {
            if (!valid[t]) continue;
            uint32_t before = 0;
            for (uint32_t o = 0; o < ne; ++o)
                if (o != t && valid[o] && (E[o].n != E[t].n ? E[o].n < E[t].n : dlexless(E[o], E[t]))) ++before;
            if (before < max_cuts) out[(size_t)q * max_cuts + before] = E[t];
            ++kept;
        }
        for (int off = 16; off; off >>= 1) kept += __shfl_xor_sync(0xFFFFFFFFu, kept, off);
        if (lane == 0) out_cnt[q] = kept < max_cuts ? kept : max_cuts;
        __syncwarp();
    }
}

__global__ void init_pi_cuts(const uint32_t *pis, uint32_t n, GCut *P, uint32_t *cnt, uint32_t C) {
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    P[(size_t)pis[i] * C].n = 1;
    P[(size_t)pis[i] * C].leaf[0] = pis[i];
    cnt[pis[i]] = 1;
}

inline const char *ck(cudaError_t e) { return e == cudaSuccess ? nullptr : cudaGetErrorString(e); }

}  // namespace

uint32_t gpu_cuts_max_C() { return CMAX; }

// Host side: level lists (Eq. 2 enumeration levels) are built by the caller.
const char *gpu_common_cuts(const uint32_t *d_f0, const uint32_t *d_f1, uint32_t N,
                            const std::vector<uint32_t> &fanout, const std::vector<uint32_t> &level,
                            const std::vector<uint32_t> &repr_of, const std::vector<uint32_t> &pis_needed,
                            const std::vector<std::vector<uint32_t>> &el_lists, const std::vector<uint32_t> &repr,
                            const std::vector<uint32_t> &member, uint32_t k_l, uint32_t C, int pass, uint32_t max_cuts,
                            void *stream, int num_sms, std::vector<uint32_t> &cut_counts,
                            std::vector<uint32_t> &cut_leaves_flat) {
    cudaStream_t st = (cudaStream_t)stream;
    const char *e = nullptr;
    uint32_t *d_fanout = nullptr, *d_level = nullptr, *d_repr_of = nullptr, *d_cnt = nullptr, *d_nodes = nullptr;
    uint32_t *d_repr = nullptr, *d_member = nullptr, *d_ocnt = nullptr;
    GCut *d_P = nullptr, *d_out = nullptr;
    const uint32_t npairs = (uint32_t)repr.size();
    size_t total_nodes = 0;
    for (auto &l : el_lists) total_nodes += l.size();
    std::vector<uint32_t> flat;
    flat.reserve(total_nodes);
    for (auto &l : el_lists) flat.insert(flat.end(), l.begin(), l.end());
    auto fin = [&]() {
        cudaFree(d_fanout); cudaFree(d_level); cudaFree(d_repr_of); cudaFree(d_cnt); cudaFree(d_nodes);
        cudaFree(d_repr); cudaFree(d_member); cudaFree(d_ocnt); cudaFree(d_P); cudaFree(d_out);
    };
#define CK(x)                 \
    do {                      \
        if ((e = ck(x))) {    \
            fin();            \
            return e;         \
        }                     \
    } while (0)
    CK(cudaMalloc(&d_fanout, sizeof(uint32_t) * N));
    CK(cudaMalloc(&d_level, sizeof(uint32_t) * N));
    CK(cudaMalloc(&d_repr_of, sizeof(uint32_t) * N));
    CK(cudaMalloc(&d_cnt, sizeof(uint32_t) * N));
    CK(cudaMalloc(&d_nodes, sizeof(uint32_t) * (flat.size() + 1)));
    CK(cudaMalloc(&d_repr, sizeof(uint32_t) * (npairs + 1)));
    CK(cudaMalloc(&d_member, sizeof(uint32_t) * (npairs + 1)));
    CK(cudaMalloc(&d_ocnt, sizeof(uint32_t) * (npairs + 1)));
    CK(cudaMalloc(&d_P, sizeof(GCut) * (size_t)N * C));
    CK(cudaMalloc(&d_out, sizeof(GCut) * ((size_t)npairs * max_cuts + 1)));
    CK(cudaMemcpyAsync(d_fanout, fanout.data(), sizeof(uint32_t) * N, cudaMemcpyHostToDevice, st));
    CK(cudaMemcpyAsync(d_level, level.data(), sizeof(uint32_t) * N, cudaMemcpyHostToDevice, st));
    CK(cudaMemcpyAsync(d_repr_of, repr_of.data(), sizeof(uint32_t) * N, cudaMemcpyHostToDevice, st));
    CK(cudaMemsetAsync(d_cnt, 0, sizeof(uint32_t) * N, st));
    if (!flat.empty()) CK(cudaMemcpyAsync(d_nodes, flat.data(), sizeof(uint32_t) * flat.size(), cudaMemcpyHostToDevice, st));
    if (npairs) {
        CK(cudaMemcpyAsync(d_repr, repr.data(), sizeof(uint32_t) * npairs, cudaMemcpyHostToDevice, st));
        CK(cudaMemcpyAsync(d_member, member.data(), sizeof(uint32_t) * npairs, cudaMemcpyHostToDevice, st));
    }
    // P(pi) = {{pi}} (Alg. 2 l.4-5)
    if (!pis_needed.empty()) {
        uint32_t *d_pis = nullptr;
        CK(cudaMalloc(&d_pis, sizeof(uint32_t) * pis_needed.size()));
        e = ck(cudaMemcpyAsync(d_pis, pis_needed.data(), sizeof(uint32_t) * pis_needed.size(), cudaMemcpyHostToDevice, st));
        if (!e) {
            init_pi_cuts<<<(unsigned)((pis_needed.size() + 255) / 256), 256, 0, st>>>(d_pis, (uint32_t)pis_needed.size(), d_P,
                                                                                     d_cnt, C);
            e = ck(cudaGetLastError());
        }
        if (!e) e = ck(cudaStreamSynchronize(st));
        cudaFree(d_pis);
        if (e) {
            fin();
            return e;
        }
    }
    const size_t smem_lvl = WPB * level_smem_per_warp();
    CK(cudaFuncSetAttribute(cut_level_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_lvl));
    size_t off = 0;
    for (auto &l : el_lists) {
        if (l.empty()) continue;
        const uint32_t n = (uint32_t)l.size();
        const unsigned grid = (unsigned)std::min<uint64_t>((uint64_t)num_sms * 2, (n + WPB - 1) / WPB);
        cut_level_kernel<<<grid, WPB * 32, smem_lvl, st>>>(d_nodes + off, n, d_f0, d_f1, d_fanout, d_level, d_repr_of,
                                                            d_P, d_cnt, k_l, C, pass);
        CK(cudaGetLastError());
        off += n;
    }
    if (npairs) {
        const size_t smem_c = WPB * (sizeof(GCut) * (CMAX * CMAX) + sizeof(uint32_t) * (CMAX * CMAX));
        CK(cudaFuncSetAttribute(common_cut_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_c));
        const unsigned grid = (unsigned)std::min<uint64_t>((uint64_t)num_sms * 2, (npairs + WPB - 1) / WPB);
        common_cut_kernel<<<grid, WPB * 32, smem_c, st>>>(d_repr, d_member, npairs, d_P, d_cnt, k_l, C, max_cuts, d_out,
                                                           d_ocnt);
        CK(cudaGetLastError());
    }
    cut_counts.assign(npairs, 0);
    std::vector<GCut> out((size_t)npairs * max_cuts);
    if (npairs) {
        CK(cudaMemcpyAsync(cut_counts.data(), d_ocnt, sizeof(uint32_t) * npairs, cudaMemcpyDeviceToHost, st));
        CK(cudaMemcpyAsync(out.data(), d_out, sizeof(GCut) * out.size(), cudaMemcpyDeviceToHost, st));
    }
    CK(cudaStreamSynchronize(st));
    cut_leaves_flat.clear();
    for (uint32_t q = 0; q < npairs; ++q)
        for (uint32_t t = 0; t < cut_counts[q]; ++t) {
            const GCut &g = out[(size_t)q * max_cuts + t];
            cut_leaves_flat.push_back(g.n);
            cut_leaves_flat.insert(cut_leaves_flat.end(), g.leaf, g.leaf + g.n);
        }
    fin();
#undef CK
    return nullptr;
}

}  // namespace cec
