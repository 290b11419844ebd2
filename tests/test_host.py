"""CPU tests of the C-ABI library: it loads, exports every symbol include/cec.h declares, and its
host logic (validation, supports, routing, windows, merging, sharding, pext) behaves as the paper
and SURVEY.md §8 say. No compute call runs here (no GPU); simulation calls must refuse loudly."""
import ctypes
import os
import re

import numpy as np
import pytest

import paper_conf_dac_liuy25_b200 as pkg
from paper_conf_dac_liuy25_b200 import capi
from workloads import Builder, c1_add8, c2_mul12, c5_big

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def host_ctx(aig, **kw):
    kw.setdefault("device", -1)
    return capi.Context.from_aig(aig, **kw)


def test_exports_match_header():
    hdr = open(os.path.join(ROOT, "include", "cec.h")).read()
    declared = set(re.findall(r"\b(cec_[a-z0-9_]+)\s*\(", hdr))
    assert declared == set(capi.EXPORTS), declared ^ set(capi.EXPORTS)
    for name in declared:
        assert hasattr(capi.lib, name)  # dlsym succeeds
    assert capi.cec_abi_version() == 2


def test_opts_layout_and_defaults():
    o = capi.cec_default_opts()
    assert (o.device, o.rank, o.world, o.k_max, o.k_s, o.merge, o.engine) == (0, 0, 1, 32, 0, 1, 0)
    assert ctypes.sizeof(capi.CecOpts) == 4 * 3 + 4 + 8 + 8 + 4 * 4 + 8 * 6


def test_validation_rejects_non_topological():
    fan = np.array([[2, 8]], dtype=np.uint32)  # AND id 3 (I=2) reading id 4
    with pytest.raises(capi.CecError) as e:
        capi.cec_load_aig(2, fan, np.array([6], np.uint32), capi.cec_default_opts(device=-1))
    assert e.value.status == capi.CEC_E_AIG
    with pytest.raises(capi.CecError) as e:
        capi.cec_load_aig(2, fan, np.array([6], np.uint32), capi.cec_default_opts(device=-1, k_max=64))
    assert e.value.status == capi.CEC_E_ARG


def test_no_cpu_fallback():
    m = c1_add8()
    ctx = host_ctx(m.aig)
    with pytest.raises(capi.CecError) as e:
        ctx.sim_exhaustive(m.lit_a, m.lit_b)
    assert e.value.status == capi.CEC_E_CUDA
    with pytest.raises(capi.CecError) as e:
        ctx.check_local_cuts(m.lit_a[:1], m.lit_b[:1], [0, 2], [1, 9])
    assert e.value.status == capi.CEC_E_CUDA


def test_supports_C1():
    m = c1_add8()
    ctx = host_ctx(m.aig)
    for j in range(8):
        S = capi.cec_pair_support(ctx.handle, int(m.lit_a[j]), int(m.lit_b[j]))
        assert S == list(range(1, j + 2)) + list(range(9, 9 + j + 1))  # {a_0..a_j, b_0..b_j}
    assert ctx.pair_k(int(m.lit_a[8]), int(m.lit_b[8])) == 16


def test_plan_C1_single_window():
    m = c1_add8()
    ctx = host_ctx(m.aig)
    plan = capi.cec_plan_exhaustive(ctx.handle, m.lit_a, m.lit_b)
    info = capi.cec_plan_info(plan)
    w = capi.cec_plan_window(plan, 0)
    assert info["num_windows"] == 1 and info["max_k"] == 16
    nontrivial = [p for p in range(9) if m.lit_a[p] != m.lit_b[p]]  # strashed-identical pairs need no sim
    assert w["inputs"] == list(range(1, 17)) and sorted(w["pairs"]) == nontrivial
    assert info["node_patterns"] == w["num_nodes"] * (1 << 16)
    # the window is exactly the ANDs in the TFI of the PO pairs (KS leaves unused prefix P terms)
    I, fan = m.aig.num_pis, m.aig.fanins
    seen, todo = set(), [int(x) >> 1 for p in nontrivial for x in (m.lit_a[p], m.lit_b[p])]
    while todo:
        v = todo.pop()
        if v in seen or v <= I:
            continue
        seen.add(v)
        todo += [int(fan[v - I - 1, 0]) >> 1, int(fan[v - I - 1, 1]) >> 1]
    assert w["num_nodes"] == len(seen)
    capi.cec_plan_free(plan)


def merge_example_aig():
    """windows with inputs {a,b}, {a,b,c}, {a,c}, {a,e}, {a,f}; ids a..f = 1..6.
    (The printed list has four windows for "five"; {a,c} is the reading-Q10 fifth window.)"""
    bd = Builder(6, strash=False)
    a, b, c, d, e, f = (bd.pi(i) for i in range(6))
    ab = bd.raw_and(a, b)
    abc = bd.raw_and(ab, c)
    ac = bd.raw_and(a, c)
    ae = bd.raw_and(a, e)
    af = bd.raw_and(a, f)
    aig = bd.finish([ab, abc, ac, ae, af])
    # pairs (node, a): support = the node's support
    la = [ab, abc, ac, ae, af]
    lb = [a] * 5
    return aig, la, lb


def test_window_merging_paper_example():
    aig, la, lb = merge_example_aig()
    ctx = host_ctx(aig, k_s=3)
    plan = capi.cec_plan_exhaustive(ctx.handle, la, lb)
    groups = sorted(capi.cec_plan_window(plan, w)["inputs"] for w in range(capi.cec_plan_info(plan)["num_windows"]))
    assert groups == [[1, 2, 3], [1, 5, 6]]  # "the first three and the last two are merged"
    capi.cec_plan_free(plan)
    ctx2 = host_ctx(aig, k_s=3, merge=capi.CEC_MERGE_OFF)
    plan = capi.cec_plan_exhaustive(ctx2.handle, la, lb)
    assert capi.cec_plan_info(plan)["num_windows"] == 5
    capi.cec_plan_free(plan)


def test_routing_k_max_and_trivial_pairs():
    m = c1_add8()
    ctx = host_ctx(m.aig, k_max=10)
    plan = capi.cec_plan_exhaustive(ctx.handle, m.lit_a, m.lit_b)
    info = capi.cec_plan_info(plan)
    assert info["max_k"] <= 10
    ks = [ctx.pair_k(int(a), int(b)) for a, b in zip(m.lit_a, m.lit_b)]
    simulated = sum(len(capi.cec_plan_window(plan, w)["pairs"]) for w in range(info["num_windows"]))
    assert simulated == sum(1 for k, a, b in zip(ks, m.lit_a, m.lit_b) if k <= 10 and a != b)
    capi.cec_plan_free(plan)


def test_c5_plan_one_window_per_copy():
    m = c5_big(copies=8, n_random=6, n_bugs=2)
    ctx = host_ctx(m.aig)
    plan = capi.cec_plan_exhaustive(ctx.handle, m.lit_a, m.lit_b)
    info = capi.cec_plan_info(plan)
    assert info["num_windows"] == 8 and info["max_k"] == 24
    W = 0
    for w in range(8):
        win = capi.cec_plan_window(plan, w)
        c = (win["inputs"][0] - 1) // 24
        assert win["inputs"] == list(range(24 * c + 1, 24 * c + 25))
        W += win["num_nodes"] << 24
    assert W == info["node_patterns"]
    capi.cec_plan_free(plan)


def test_shard_range_partition():
    for n in [0, 1, 7, 2048, 16384, 10**9 + 7]:
        for G in [1, 2, 3, 4, 8]:
            rs = [capi.cec_shard_range(n, g, G) for g in range(G)]
            assert rs[0][0] == 0 and rs[-1][1] == n
            assert all(rs[g][1] == rs[g + 1][0] for g in range(G - 1))
            assert max(e - b for b, e in rs) - min(e - b for b, e in rs) <= 1


def test_pext():
    assert capi.cec_pext64(6, 0b110) == 3  # survey vector V3
    rng = np.random.default_rng(0)
    for _ in range(200):
        v, m = int(rng.integers(0, 2**63)), int(rng.integers(0, 2**63))
        want, j = 0, 0
        for b in range(64):
            if (m >> b) & 1:
                want |= ((v >> b) & 1) << j
                j += 1
        assert capi.cec_pext64(v, m) == want


def test_jit_codegen_compiles_for_sm100a_host_only(monkeypatch):
    """The JIT engine's NVRTC path runs on the host (no GPU needed): one kernel per distinct window
    structure; C5's 256 copies share 3 random + 1 mul12 + bug-variant structures. Structures too
    small to fill the GPU alone are compiled together into one bundle kernel."""
    m = c5_big(copies=12, n_random=8, n_bugs=2, rand_pis=12, rand_ands=300, mul_n=6)
    n_struct = len(set(m.meta["types"]))
    monkeypatch.setenv("CEC_NO_BUNDLE", "1")
    ctx = host_ctx(m.aig, engine=capi.CEC_ENGINE_JIT, k_s=12)  # merge inside a copy, never across
    plan = capi.cec_plan_exhaustive(ctx.handle, m.lit_a, m.lit_b)
    st = ctx.stats()
    assert st["jit_windows"] == 12 and st["jit_kernels"] == n_struct
    capi.cec_plan_free(plan)
    monkeypatch.delenv("CEC_NO_BUNDLE")
    plan = capi.cec_plan_exhaustive(ctx.handle, m.lit_a, m.lit_b)
    st = ctx.stats()
    assert st["jit_windows"] == 12 and st["jit_kernels"] == 1  # every structure in one bundle
    capi.cec_plan_free(plan)
    # interpreter only: no JIT
    ctx2 = host_ctx(m.aig, engine=capi.CEC_ENGINE_INTERP)
    plan = capi.cec_plan_exhaustive(ctx2.handle, m.lit_a, m.lit_b)
    assert ctx2.stats()["jit_windows"] == 0
    capi.cec_plan_free(plan)


@pytest.mark.parametrize("world", [2, 4, 8])
def test_small_windows_go_whole_to_one_rank_lpt(world):
    """SURVEY.md §8(e) "tiny windows": windows with fewer slices than ranks are not split but given
    whole to one rank by LPT over their node-words, so per-rank work stays balanced; every window's
    patterns are still covered exactly once (per-rank W adds up to the whole)."""
    from workloads import circuits
    m = circuits.c3_rand(n_blocks=40, block_ands=200, num_pis=256, n_internal=300, n_near=8,
                         k_dist=((40, 10, 14),))
    Ws = []
    for r in range(world):
        ctx = host_ctx(m.aig, rank=r, world=world, engine=capi.CEC_ENGINE_INTERP, merge=capi.CEC_MERGE_OFF)
        plan = capi.cec_plan_exhaustive(ctx.handle, m.lit_a, m.lit_b)
        st = ctx.stats()
        Ws.append(st["node_patterns"])
        W_all = st["node_patterns_all"]
        capi.cec_plan_free(plan)
        ctx.close()
    assert sum(Ws) == W_all
    assert max(Ws) <= 1.6 * W_all / world  # balanced (one-rank-takes-all would be `world` x)


def test_peer_mode_needs_a_device_and_world():
    """cec_peer_export (include/cec.h): a host-only context has no device memory to share."""
    m = c1_add8()
    ctx = capi.Context.from_aig(m.aig, device=-1, rank=0, world=2)
    with pytest.raises(capi.CecError) as e:
        capi.cec_peer_export(ctx.handle)
    assert e.value.status == capi.CEC_E_CUDA
    with pytest.raises(capi.CecError) as e:
        capi.cec_peer_import(ctx.handle, [bytes(128), bytes(128)])
    assert e.value.status == capi.CEC_E_CUDA
    with pytest.raises(capi.CecError) as e:  # host barriers only for a connected peer context
        capi.cec_peer_host_barrier(ctx.handle, lambda: None)
    assert e.value.status == capi.CEC_E_STATE


def test_merge_never_exceeds_enumeration_limit():
    """merging was bounded by min(k_s, k_max) only, so with k_max = 63 two
    30-input windows could merge into a 45-input window whose 2^40 slices do not fit the u32 work
    items (the tail was never simulated: a false EQ). The merge threshold is now also capped at the
    enumeration limit (41 inputs, cec_host.cpp MAX_K_ENUM) that single pairs already obey."""
    bd = Builder(60, strash=False)

    def chain(lo, hi):
        x = bd.pi(lo)
        for i in range(lo + 1, hi):
            x = bd.raw_and(x, bd.pi(i))
        return x

    f1, f2 = chain(0, 30), chain(15, 45)  # supports {1..30}, {16..45}: union of 45 PIs
    aig = bd.finish([f1, f2])
    for k_s in (0, 45, 63):
        ctx = host_ctx(aig, k_max=63, k_s=k_s, engine=capi.CEC_ENGINE_INTERP)
        plan = capi.cec_plan_exhaustive(ctx.handle, [f1, f2], [0, 0])
        info = capi.cec_plan_info(plan)
        assert info["num_windows"] == 2 and info["max_k"] == 30, (k_s, info)
        capi.cec_plan_free(plan)
        ctx.close()
    # a pair whose own support exceeds the limit stays UNDECIDED (never enumerated)
    f3 = chain(0, 42)
    aig = bd.finish([f3])
    ctx = host_ctx(aig, k_max=63, engine=capi.CEC_ENGINE_INTERP)
    plan = capi.cec_plan_exhaustive(ctx.handle, [f3], [0])
    assert capi.cec_plan_info(plan)["num_windows"] == 0
    capi.cec_plan_free(plan)
    ctx.close()


def test_binding_rejects_mismatched_pair_arrays():
    """the binding passes n = len(lit_a) to the C side, which reads n entries of every
    per-pair array; mismatched lengths (or a cut_off that is not the CSR of the leaves) must be
    refused before the call instead of reading past a numpy buffer."""
    m = c1_add8()
    ctx = host_ctx(m.aig)
    with pytest.raises(ValueError):
        ctx.sim_exhaustive(m.lit_a, m.lit_b[:-1])
    with pytest.raises(ValueError):
        capi.cec_plan_exhaustive(ctx.handle, m.lit_a[:3], m.lit_b)
    for off, leaves in (([0], [1, 9]), ([0, 2, 2], [1, 9]), ([0, 3], [1, 9]), ([1, 2], [1, 9])):
        with pytest.raises(ValueError):
            ctx.check_local_cuts(m.lit_a[:1], m.lit_b[:1], off, leaves)
    with pytest.raises(ValueError):
        ctx.check_local_cuts(m.lit_a[:2], m.lit_b[:2], [0, 2, 1], [1, 9])
    with pytest.raises(ValueError):
        capi.cec_local_pass(ctx.handle, [1, 2], [3], [0, 0], 4, 4, 0, 4)
    # well-formed arguments still reach the C side (which refuses: no device, no CPU fallback)
    with pytest.raises(capi.CecError):
        ctx.check_local_cuts(m.lit_a[:1], m.lit_b[:1], [0, 2], [1, 9])


@pytest.mark.parametrize("world", [1, 3, 8])
def test_free_warp_partition_host_plans(world):
    """Free-warp JIT kernels (single small structures, round 2): the planner cuts each group's
    slices into one contiguous range per warp of the launch grid and checks (CEC_E_STATE otherwise)
    that the items tile every window's slice range exactly once; per-rank work still adds up to the
    whole under pattern-space sharding (C2's single window, and a reduced C5 with mul copies)."""
    from workloads import circuits
    for m in (circuits.c2_mul12(10), c5_big(copies=6, n_random=2, n_bugs=1, rand_pis=12, rand_ands=300, mul_n=6)):
        Ws, W_all = [], None
        for r in range(world):
            ctx = host_ctx(m.aig, rank=r, world=world, engine=capi.CEC_ENGINE_JIT)
            plan = capi.cec_plan_exhaustive(ctx.handle, m.lit_a, m.lit_b)
            st = ctx.stats()
            assert st["jit_windows"] >= 1
            Ws.append(st["node_patterns"])
            W_all = st["node_patterns_all"]
            capi.cec_plan_free(plan)
            ctx.close()
        assert sum(Ws) == W_all


def test_reload_aig_replaces_the_miter_and_rejects_bad_arrays():
    """cec_reload_aig (include/cec.h): the next miter version in the same context gives exactly what
    a fresh context of that AIG gives; a malformed AIG is rejected and leaves the context unchanged."""
    a, b = c1_add8(), c2_mul12()
    ctx = capi.Context.from_aig(a.aig, device=-1)
    sa = [ctx.pair_k(int(x), int(y)) for x, y in zip(a.lit_a, a.lit_b)]
    ctx.reload(b.aig, k_max=24)
    fresh = capi.Context.from_aig(b.aig, device=-1)
    for x, y in zip(b.lit_a, b.lit_b):
        assert capi.cec_pair_support(ctx.handle, int(x), int(y)) == capi.cec_pair_support(fresh.handle, int(x), int(y))
    assert ctx.opts is not None and ctx.num_ands == b.aig.num_ands
    bad = np.array(b.aig.fanins, dtype=np.uint32).copy()
    bad[0, 0] = 2 * (1 + b.aig.num_pis + 5)  # fanin id above its own id
    with pytest.raises(capi.CecError) as e:
        capi.cec_reload_aig(ctx.handle, b.aig.num_pis, bad, b.aig.pos)
    assert e.value.status == capi.CEC_E_AIG
    for x, y in zip(b.lit_a[:4], b.lit_b[:4]):  # unchanged: still the valid C2 AIG
        assert capi.cec_pair_support(ctx.handle, int(x), int(y)) == capi.cec_pair_support(fresh.handle, int(x), int(y))
    ctx.reload(a.aig)
    assert [ctx.pair_k(int(x), int(y)) for x, y in zip(a.lit_a, a.lit_b)] == sa
