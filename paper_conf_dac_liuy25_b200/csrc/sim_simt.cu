// sim_simt.cu — the paper's own exhaustive-simulation design (Alg. 1) on B200,
// kept as an engine (CEC_ENGINE_SIMT) to measure the prior-art design on the same hardware.
//
// A simulation table `simt` in HBM holds E = 2^e words per window node and input (Alg. 1 l.1-3,
// E the largest power of two with E x rows <= M). Round r covers words [rE, (r+1)E) of every
// window still longer than rE (l.5-6); in each round the projection segments of the inputs are
// written (l.9), then every topological level is one launch over all (node, word) items of that
// level in all active windows (l.10-11, "level-wise parallel"), and the pair segments are
// XOR-compared at the end of the round (l.12-14) with the minimum mismatching index kept
// (canonical CEX). B200 care: rows are 16-byte aligned and every thread moves
// 4 words with 128-bit loads/stores, consecutive threads on consecutive words (coalesced).
// Its bound is HBM: 12 B per node per 32 patterns (2 reads + 1 write of a u32 word).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <vector>

#include "cec_internal.hpp"

namespace cec {
namespace {

__device__ __forceinline__ uint32_t sproj(uint32_t j, uint64_t w) {
    switch (j) {
        case 0: return 0xAAAAAAAAu;
        case 1: return 0xCCCCCCCCu;
        case 2: return 0xF0F0F0F0u;
        case 3: return 0xFF00FF00u;
        case 4: return 0xFFFF0000u;
        default: return 0u - (uint32_t)((w >> (j - 5)) & 1u);
    }
}

// inputs: {row, window, j, 0}
__global__ void simt_inputs(const uint4 *__restrict__ ins, uint32_t n, const unsigned long long *__restrict__ ttw,
                            uint64_t r, uint32_t E, uint4 *simt) {
    const uint32_t q4 = E / 4;
    const uint64_t total = (uint64_t)n * q4;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < total; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint4 d = ins[i / q4];
        const uint64_t w0 = r * E + 4 * (i % q4);
        if (w0 >= ttw[d.y]) continue;
        simt[(uint64_t)d.x * q4 + i % q4] = make_uint4(sproj(d.z, w0), sproj(d.z, w0 + 1), sproj(d.z, w0 + 2), sproj(d.z, w0 + 3));
    }
}

// nodes of one level: {row_out, row_f0 | c0 << 31, row_f1 | c1 << 31, window}
__global__ void simt_level(const uint4 *__restrict__ nodes, uint32_t n, const unsigned long long *__restrict__ ttw,
                           uint64_t r, uint32_t E, uint4 *simt) {
    const uint32_t q4 = E / 4;
    const uint64_t total = (uint64_t)n * q4;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < total; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint4 d = nodes[i / q4];
        const uint32_t q = (uint32_t)(i % q4);
        if (r * E + 4ull * q >= ttw[d.w]) continue;
        const uint32_t m0 = 0u - (d.y >> 31), m1 = 0u - (d.z >> 31);
        const uint4 a = simt[(uint64_t)(d.y & 0x7FFFFFFFu) * q4 + q];
        const uint4 b = simt[(uint64_t)(d.z & 0x7FFFFFFFu) * q4 + q];
        simt[(uint64_t)d.x * q4 + q] =
            make_uint4((a.x ^ m0) & (b.x ^ m1), (a.y ^ m0) & (b.y ^ m1), (a.z ^ m0) & (b.z ^ m1), (a.w ^ m0) & (b.w ^ m1));
    }
}

// pairs: {row_a | ca << 31, row_b | cb << 31, window, cmp index}
__global__ void simt_compare(const uint4 *__restrict__ pairs, uint32_t n, const unsigned long long *__restrict__ ttw,
                             uint64_t r, uint32_t E, const uint4 *__restrict__ simt, unsigned long long *first) {
    const uint32_t q4 = E / 4;
    const uint64_t total = (uint64_t)n * q4;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < total; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint4 d = pairs[i / q4];
        const uint32_t q = (uint32_t)(i % q4);
        const uint64_t w0 = r * E + 4ull * q, tw = ttw[d.z];
        if (w0 >= tw) continue;
        const uint32_t m = 0u - ((d.x ^ d.y) >> 31);
        const uint4 a = simt[(uint64_t)(d.x & 0x7FFFFFFFu) * q4 + q];
        const uint4 b = simt[(uint64_t)(d.y & 0x7FFFFFFFu) * q4 + q];
        const uint32_t x[4] = {a.x ^ b.x ^ m, a.y ^ b.y ^ m, a.z ^ b.z ^ m, a.w ^ b.w ^ m};
        for (uint32_t t = 0; t < 4 && w0 + t < tw; ++t)
            if (x[t]) {
                atomicMin(&first[d.w], ((w0 + t) << 5) + (unsigned long long)(__ffs(x[t]) - 1));
                break;
            }
    }
}

inline const char *ck(cudaError_t e) { return e == cudaSuccess ? nullptr : cudaGetErrorString(e); }

}  // namespace

const char *launch_simt(const SimtPlan &S, unsigned long long *first, uint32_t ncmp, void *stream, int num_sms,
                        uint32_t *launches) {
    cudaStream_t st = (cudaStream_t)stream;
    const char *e;
    if ((e = ck(cudaMemsetAsync(first, 0xFF, sizeof(unsigned long long) * (ncmp ? ncmp : 1), st)))) return e;
    if ((e = ck(cudaMemsetAsync(S.d_simt, 0, sizeof(uint4) * (S.E / 4), st)))) return e;  // row 0 = constant 0
    const int T = 256;
    auto grid = [&](uint64_t items) {
        return (unsigned)std::max<uint64_t>(1, std::min<uint64_t>((uint64_t)num_sms * 16, (items + T - 1) / T));
    };
    uint32_t nl = 0;
    for (uint64_t r = 0; r < S.rounds; ++r) {
        // windows still active in round r: ttw > rE; their inputs/levels/pairs are filtered in-kernel
        simt_inputs<<<grid((uint64_t)S.n_inputs * (S.E / 4)), T, 0, st>>>(S.d_inputs, S.n_inputs, S.d_ttw, r, S.E, S.d_simt);
        ++nl;
        for (size_t l = 0; l + 1 < S.level_off.size(); ++l) {
            const uint32_t n = S.level_off[l + 1] - S.level_off[l];
            if (!n) continue;
            simt_level<<<grid((uint64_t)n * (S.E / 4)), T, 0, st>>>(S.d_nodes + S.level_off[l], n, S.d_ttw, r, S.E, S.d_simt);
            ++nl;
        }
        simt_compare<<<grid((uint64_t)S.n_pairs * (S.E / 4)), T, 0, st>>>(S.d_pairs, S.n_pairs, S.d_ttw, r, S.E, S.d_simt,
                                                                         first);
        ++nl;
        if ((e = ck(cudaGetLastError()))) return e;
    }
    if (launches) *launches = nl;
    return nullptr;
}

}  // namespace cec
