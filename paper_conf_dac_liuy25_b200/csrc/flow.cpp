// flow.cpp — C-ABI entries of the GPU steps around the hot path:
//   cec_sim_classes (NEXT-2, PAPER.md:41/:61/:183/:187): partial simulation -> equivalence classes ->
//                   candidate pairs, kernels in classes_gpu.cu;
//   cec_reduce      (NEXT-3, PAPER.md:61/:185/:187): miter reduction. Validates the merge list,
//                   builds the topological batch schedule on the host (O(N): batch(member) =
//                   batch(repr) + 1, batch(AND) = 1 + max over fanins) and runs reduce_gpu.cu on
//                   the context's device copy of the AIG.
#include <chrono>
#include <cstring>
#include <memory>
#include <string>
#include <vector>

#include "cec_ctx.hpp"

extern "C" cec_status cec_reduce(cec_ctx *c, uint32_t num_subst, const uint32_t *member, const uint32_t *repr_lit,
                                 uint32_t *new_num_ands, uint32_t *new_fanin_lits, uint32_t *image_out,
                                 uint32_t num_lits, uint32_t *lits) {
    if (!c) return CEC_E_ARG;
    if ((num_subst && (!member || !repr_lit)) || !new_num_ands || (c->A && !new_fanin_lits) || (num_lits && !lits)) {
        c->err = "null argument";
        return CEC_E_ARG;
    }
    const auto t0 = std::chrono::steady_clock::now();
    const uint32_t N = c->N();
    constexpr uint32_t NONE = 0xFFFFFFFFu;
    std::vector<uint32_t> sub(N, NONE);
    for (uint32_t q = 0; q < num_subst; ++q) {
        const uint32_t m = member[q], r = repr_lit[q];
        if (m <= c->I || m >= N || (r >> 1) >= m || sub[m] != NONE) {
            c->err = "merge " + std::to_string(q) + ": member must be an AND id, listed once, above its representative";
            return CEC_E_ARG;
        }
        sub[m] = r;
    }
    for (uint32_t i = 0; i < num_lits; ++i)
        if ((lits[i] >> 1) >= N) {
            c->err = "literal out of range";
            return CEC_E_ARG;
        }
    if (c->host_only) {
        c->err = "host-only context: no CUDA device (no CPU fallback)";
        return CEC_E_CUDA;
    }
    // topological batch schedule
    std::vector<uint32_t> batch(N, 0);
    uint32_t nb = 0;
    for (uint32_t id = c->I + 1; id < N; ++id) {
        batch[id] = sub[id] != NONE ? batch[sub[id] >> 1] + 1
                                    : 1 + std::max(batch[c->f0[id] >> 1], batch[c->f1[id] >> 1]);
        nb = std::max(nb, batch[id]);
    }
    std::vector<uint32_t> off(nb + 2, 0), ids(c->A);
    for (uint32_t id = c->I + 1; id < N; ++id) ++off[batch[id] + 1];
    for (size_t b = 1; b < off.size(); ++b) off[b] += off[b - 1];
    {
        std::vector<uint32_t> fill(off.begin(), off.end());
        for (uint32_t id = c->I + 1; id < N; ++id) ids[fill[batch[id]]++] = id;
    }
    // batch 0 holds no AND; drop it from the offsets
    std::vector<uint32_t> boff(off.begin() + 1, off.end());
    cec_status st = cec_ensure_device_aig(c);
    if (st != CEC_OK) return st;
    std::vector<uint32_t> fan, image;
    uint32_t nl = 0;
    if (!c->devpool) c->devpool = std::make_shared<DevPool>();
    float kms = 0.f;
    const float host_ms = std::chrono::duration<float, std::milli>(std::chrono::steady_clock::now() - t0).count();
    if (const char *e = gpu_reduce(c->d_f0, c->d_f1, c->I, N, sub, ids, boff, c->stream, c->num_sms, c->devpool.get(),
                                   fan, image, &nl, &kms)) {
        c->err = std::string("CUDA: ") + e + " (miter reduction)";
        return CEC_E_CUDA;
    }
    *new_num_ands = (uint32_t)(fan.size() / 2);
    if (!fan.empty()) std::memcpy(new_fanin_lits, fan.data(), 4 * fan.size());
    if (image_out) std::memcpy(image_out, image.data(), 4 * (size_t)N);
    for (uint32_t i = 0; i < num_lits; ++i) lits[i] = image[lits[i] >> 1] ^ (lits[i] & 1u);
    c->stats.num_launches = nl;
    c->stats.kernel_ms = kms;
    c->stats.host_prep_ms = host_ms;
    return CEC_OK;
}

extern "C" cec_status cec_sim_classes(cec_ctx *c, uint32_t num_words, uint64_t seed, uint32_t num_pattern_words,
                                      const uint32_t *pi_words, uint32_t cap, uint32_t *num_pairs_out,
                                      uint32_t *repr_out, uint32_t *member_out, uint8_t *phase_out) {
    if (!c) return CEC_E_ARG;
    if (!num_pairs_out || (cap && (!repr_out || !member_out || !phase_out)) || (num_pattern_words && !pi_words) ||
        num_words + (uint64_t)num_pattern_words == 0) {
        c->err = "null argument or no patterns";
        return CEC_E_ARG;
    }
    if (c->host_only) {
        c->err = "host-only context: no CUDA device (no CPU fallback)";
        return CEC_E_CUDA;
    }
    cec_status st = cec_ensure_device_aig(c);
    if (st != CEC_OK) return st;
    std::vector<uint32_t> r, m;
    std::vector<uint8_t> ph;
    uint32_t total = 0, nl = 0;
    float kms = 0.f;
    if (!c->devpool) c->devpool = std::make_shared<DevPool>();
    if (const char *e = gpu_classes(c->d_f0, c->d_f1, c->d_level_ids, c->level_off, c->I, c->N(), num_words, seed,
                                    num_pattern_words, pi_words, cap, c->stream, c->num_sms, c->devpool.get(), &total,
                                    r, m, ph, &nl, &kms)) {
        c->err = std::string("CUDA: ") + e + " (equivalence classes)";
        return CEC_E_CUDA;
    }
    *num_pairs_out = total;
    if (!r.empty()) {
        std::memcpy(repr_out, r.data(), 4 * r.size());
        std::memcpy(member_out, m.data(), 4 * m.size());
        std::memcpy(phase_out, ph.data(), ph.size());
    }
    c->stats.num_launches = nl;
    c->stats.kernel_ms = kms;
    return CEC_OK;
}
