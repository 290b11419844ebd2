// sim_random.cu — partial random simulation of the whole AIG on the GPU (§II-B,
// :61 "the partial simulator performs simulation of random patterns for initializing the ECs",
// :183). Produces one complement-canonical 64-bit signature per node; nodes with equal signatures
// form the candidate equivalence classes whose (representative, member) pairs the exhaustive
// checker then proves or refutes.
//
// Layout: tt[id * W + w] (u32 words, W words per node, node-major) in HBM. PI words come from a
// counter-based generator (splitmix64 of seed, PI id, word), so results do not depend on launch
// shape. Levels are simulated in order, one launch per level, one thread per (node, word) of the
// level (the paper's level-wise parallelism) — this pass is HBM-bound and small
// next to the exhaustive sweep.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <vector>

#include "cec_internal.hpp"

namespace cec {
namespace {

__device__ __forceinline__ uint64_t splitmix64(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}

__global__ void rs_pis(uint32_t *tt, uint32_t I, uint32_t W, uint64_t seed) {
    const uint64_t n = (uint64_t)I * W;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t pi = 1 + i / W, w = i % W;
        tt[pi * W + w] = (uint32_t)splitmix64(seed ^ (pi << 32) ^ w);
    }
    if (blockIdx.x == 0)
        for (uint32_t w = threadIdx.x; w < W; w += blockDim.x) tt[w] = 0u;  // constant node 0
}

__global__ void rs_level(uint32_t *tt, const uint32_t *__restrict__ ids, uint32_t n, const uint32_t *__restrict__ f0,
                         const uint32_t *__restrict__ f1, uint32_t W) {
    const uint64_t total = (uint64_t)n * W;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < total;
         i += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t node = ids[i / W];
        const uint32_t w = (uint32_t)(i % W);
        const uint32_t l0 = f0[node], l1 = f1[node];
        const uint32_t a = tt[(uint64_t)(l0 >> 1) * W + w] ^ (0u - (l0 & 1u));
        const uint32_t b = tt[(uint64_t)(l1 >> 1) * W + w] ^ (0u - (l1 & 1u));
        tt[(uint64_t)node * W + w] = a & b;
    }
}

__global__ void rs_signature(const uint32_t *__restrict__ tt, uint32_t N, uint32_t W, unsigned long long *sig,
                             uint8_t *phase) {
    for (uint32_t id = blockIdx.x * blockDim.x + threadIdx.x; id < N; id += gridDim.x * blockDim.x) {
        const uint32_t *row = tt + (uint64_t)id * W;
        const uint32_t inv = 0u - (row[0] & 1u);  // canonical phase: pattern 0 evaluates to 0
        uint64_t h = 0x243F6A8885A308D3ull ^ W;
        for (uint32_t w = 0; w < W; ++w) h = splitmix64(h ^ (row[w] ^ inv));
        sig[id] = h;
        phase[id] = (uint8_t)(inv & 1u);
    }
}

inline const char *ck(cudaError_t e) { return e == cudaSuccess ? nullptr : cudaGetErrorString(e); }

}  // namespace

const char *random_sim(const uint32_t *d_f0, const uint32_t *d_f1, const uint32_t *d_level_ids,
                       const std::vector<uint32_t> &level_off, uint32_t I, uint32_t N, uint32_t W, uint64_t seed,
                       uint32_t *d_tt, unsigned long long *d_sig, uint8_t *d_phase, void *stream, int num_sms,
                       uint32_t *launches, bool pi_words_given) {
    cudaStream_t st = (cudaStream_t)stream;
    const int T = 256;
    const uint64_t grid_cap = (uint64_t)num_sms * 8;
    auto grid_for = [&](uint64_t work) { return (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(grid_cap, (work + T - 1) / T)); };
    uint32_t nl = 0;
    const char *e;
    if (!pi_words_given) {
        rs_pis<<<grid_for((uint64_t)I * W + W), T, 0, st>>>(d_tt, I, W, seed);
        ++nl;
        if ((e = ck(cudaGetLastError()))) return e;
    }
    for (size_t l = 1; l + 1 < level_off.size(); ++l) {
        const uint32_t n = level_off[l + 1] - level_off[l];
        if (!n) continue;
        rs_level<<<grid_for((uint64_t)n * W), T, 0, st>>>(d_tt, d_level_ids + level_off[l], n, d_f0, d_f1, W);
        ++nl;
        if ((e = ck(cudaGetLastError()))) return e;
    }
    rs_signature<<<grid_for(N), T, 0, st>>>(d_tt, N, W, d_sig, d_phase);
    ++nl;
    if (launches) *launches = nl;
    return ck(cudaGetLastError());
}

}  // namespace cec
