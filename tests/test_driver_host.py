"""Host logic of the CEC driver (no GPU): Eq. (1) cut enumeration on hand graphs, Table I orders,
class formation from signatures, and miter reduction preserving PO functions (checked with the
oracle's evaluator on random assignments)."""
import os

import numpy as np
import pytest

import oracle
from paper_conf_dac_liuy25_b200 import driver
from workloads import Builder, c4_dp, circuits


def test_eq1_cut_enumeration_hand_graph():
    bd = Builder(3, strash=False)
    a, b, c = bd.pi(0), bd.pi(1), bd.pi(2)
    n = bd.raw_and(a, b)      # id 4
    m = bd.raw_and(n, c)      # id 5
    aig = bd.finish([m])
    P = driver.enumerate_cuts(aig, k_l=8, C=8, pass_id=1)
    as_sets = lambda cuts: sorted(sorted(driver._bits(x)) for x in cuts)
    assert as_sets(P[4]) == [[1, 2]]
    assert as_sets(P[5]) == [[1, 2, 3], [3, 4]]   # {u|v : u in P(n)+{{n}}, v in {{c}}}
    # k_l bound: no cut above 2 leaves survives
    P2 = driver.enumerate_cuts(aig, k_l=2, C=8, pass_id=1)
    assert as_sets(P2[5]) == [[3, 4]]


def test_table1_orders():
    bd = Builder(4, strash=False)
    x = [bd.pi(i) for i in range(4)]
    n1 = bd.raw_and(x[0], x[1])
    n2 = bd.raw_and(n1, x[2])
    n3 = bd.raw_and(n2, x[3])
    aig = bd.finish([n3])
    small_level = driver.enumerate_cuts(aig, 8, 1, pass_id=1)[n3 >> 1]
    large_level = driver.enumerate_cuts(aig, 8, 1, pass_id=2)[n3 >> 1]
    assert sorted(driver._bits(small_level[0])) == [1, 2, 3, 4]     # PIs: level 0
    assert sorted(driver._bits(large_level[0])) == [4, n2 >> 1]     # highest-level leaves


@pytest.mark.gpu
def test_miter_reduction_preserves_functions():
    """The driver's reduction (GPU cec_reduce) keeps every PO function (oracle evaluator)."""
    m = circuits.random_miter(10, 200, 8, seed=3, window=24)
    # merge every B-side PO driver into its A-side partner (they are equivalent by construction)
    cur = driver.Miter(m.aig, m.lit_a, m.lit_b)
    subst = {}
    for a, b in zip(m.lit_a, m.lit_b):
        a, b = int(a), int(b)
        hi, lo = (a, b) if (a >> 1) > (b >> 1) else (b, a)
        if (hi >> 1) > m.aig.num_pis and (hi >> 1) != (lo >> 1) and (hi >> 1) not in subst:
            subst[hi >> 1] = lo ^ (hi & 1)
    red, _ = cur.reduce(subst)
    assert all(int(x) == int(y) for x, y in zip(red.lit_a, red.lit_b))
    o1, o2 = oracle.Oracle.from_aig(m.aig), oracle.Oracle.from_aig(red.aig)
    rng = np.random.default_rng(0)
    for _ in range(64):
        pis = rng.integers(0, 2, size=10).astype(np.uint8)
        for a_old, a_new in zip(m.lit_a, red.lit_a):
            assert o1.eval_lit(int(a_old), pis) == o2.eval_lit(int(a_new), pis)


def test_native_common_cuts_are_valid_cuts():
    """cec_common_cuts (C++, host-only): every returned common cut is a real cut of both roots
    (the oracle's cut validation accepts it), has <= k_l leaves in increasing id, and no pair gets
    more than max_cuts cuts."""
    from paper_conf_dac_liuy25_b200 import capi
    from workloads import c4_dp
    m = c4_dp(8)
    ctx = capi.Context.from_aig(m.aig, device=-1)
    # candidate pairs: the PO pairs whose B driver has a higher id (repr = A side)
    pairs = [(int(a) >> 1, int(b) >> 1, (int(a) ^ int(b)) & 1) for a, b in zip(m.lit_a, m.lit_b)
             if (int(a) >> 1) < (int(b) >> 1) and (int(a) >> 1) > m.aig.num_pis]
    orc = oracle.Oracle.from_aig(m.aig)
    for pass_id in range(3):
        pco, co, lv = capi.cec_common_cuts(ctx.handle, [r for r, _, _ in pairs], [x for _, x, _ in pairs], 10, 8,
                                           pass_id, 6)
        la, lb, off, leaves = [], [], [0], []
        for i, (r, mm, f) in enumerate(pairs):
            assert pco[i + 1] - pco[i] <= 6
            for t in range(int(pco[i]), int(pco[i + 1])):
                L = [int(x) for x in lv[co[t]:co[t + 1]]]
                assert 1 <= len(L) <= 10 and L == sorted(L)
                la.append(2 * r)
                lb.append(2 * mm ^ f)
                leaves += L
                off.append(len(leaves))
        assert la, "some common cuts expected"
        v = orc.check_local(la, lb, off, leaves)
        assert all(int(x) != oracle.BADCUT for x in v)


def test_pack_patterns():
    pats = [np.array([1, 0, 1], np.uint8), np.array([0, 1, 1], np.uint8)] + [np.zeros(3, np.uint8)] * 30 + \
           [np.array([1, 1, 0], np.uint8)]
    w = driver.pack_patterns(pats, 3)
    assert w.shape == (3, 2)
    assert [int(x) for x in w[:, 0]] == [0b01, 0b10, 0b11] and [int(x) for x in w[:, 1]] == [0b1, 0b1, 0]


import pytest  # noqa: E402


@pytest.mark.parametrize("case", range(10))
def test_native_common_cuts_match_cut_oracle(case):
    """cec_common_cuts (C++) == oracle/cuts.py (plain Python, exact arithmetic) cut for cut."""
    from oracle import cuts as cut_oracle
    from paper_conf_dac_liuy25_b200 import capi
    from workloads import c4_dp
    rng = np.random.default_rng(case)
    if case < 4:
        m = c4_dp(6 + 2 * case)
    else:
        m = circuits.random_miter(12, 150 + 40 * case, 10, seed=900 + case, window=24)
    aig = m.aig
    # candidate pairs: (lower id, higher id) of the PO pairs and of random node pairs
    pairs = set()
    for a, b in zip(m.lit_a, m.lit_b):
        x, y = sorted((int(a) >> 1, int(b) >> 1))
        if x < y:
            pairs.add((x, y))
    N = aig.num_nodes
    for _ in range(20):
        x, y = sorted(int(v) for v in rng.integers(1, N, size=2))
        if x < y:
            pairs.add((x, y))
    pairs = sorted(pairs)
    # a member may have one representative only
    seen, P = set(), []
    for x, y in pairs:
        if y not in seen:
            seen.add(y)
            P.append((x, y))
    k_l, C, pass_id, mc = int(rng.integers(4, 13)), int(rng.integers(2, 9)), case % 3, int(rng.integers(1, 7))
    ctx = capi.Context.from_aig(aig, device=-1)
    pco, co, lv = capi.cec_common_cuts(ctx.handle, [x for x, _ in P], [y for _, y in P], k_l, C, pass_id, mc)
    want = cut_oracle.common_cuts(aig.num_pis, aig.fanins, [x for x, _ in P], [y for _, y in P], k_l, C, pass_id, mc)
    for i in range(len(P)):
        got = [tuple(int(v) for v in lv[co[t]:co[t + 1]]) for t in range(int(pco[i]), int(pco[i + 1]))]
        assert got == want[i], (i, P[i], got, want[i])


def test_tried_pairs_follow_the_reduction():
    """the G phase's record of decided pairs is keyed by node ids of one miter version;
    after cec_reduce renumbers the ANDs each entry must denote the same functional pair (the image
    literals), and pairs whose sides collapsed are dropped."""
    from paper_conf_dac_liuy25_b200.driver import _remap_tried
    import numpy as np
    # old ids 0..9; image = new literal of each old id
    image = np.array([0, 2, 4, 6, 8, 10, 8, 13, 14, 9], np.uint32)
    tried = {(4, 5, 0),   # images 8, 10 -> (4, 5, 0)
             (4, 6, 0),   # 6 collapsed onto 4 (both image 8): dropped
             (5, 7, 1),   # 10 vs 13 ^ 1 = 12 -> (5, 6, 0)
             (3, 9, 0),   # 6 vs 9 -> (3, 4, 1)
             (8, 2, 1)}   # 14 vs 4 ^ 1 = 5 -> lower id first: (2, 7, 1)
    assert _remap_tried(tried, image) == {(4, 5, 0), (5, 6, 0), (3, 4, 1), (2, 7, 1)}


def test_cut_masks_path_equals_lists_path():
    """node_cuts' 128-bit dictionary path (csrc/cuts.cpp) and its list path (CEC_CUTS_LISTS=1) give
    identical common cuts at C4's parameters (k_l = C = 16, 64-bit datapath, all three passes)."""
    import subprocess
    import sys
    script = r"""
import hashlib, sys
sys.path.insert(0, %r)
import numpy as np
from paper_conf_dac_liuy25_b200 import capi
from workloads import c4_dp
m = c4_dp(64)
ctx = capi.Context.from_aig(m.aig, device=-1)
I = m.aig.num_pis
pairs = sorted({(min(a >> 1, b >> 1), max(a >> 1, b >> 1)) for a, b in zip(m.lit_a.tolist(), m.lit_b.tolist())
                if (a >> 1) != (b >> 1) and min(a >> 1, b >> 1) > I})
h = hashlib.sha1()
for pass_id in range(3):
    for a in capi.cec_common_cuts(ctx.handle, [p[0] for p in pairs], [p[1] for p in pairs], 16, 16, pass_id, 16):
        h.update(np.ascontiguousarray(a).tobytes())
print(h.hexdigest())
""" % os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ)
    env.pop("CEC_CUTS_LISTS", None)
    a = subprocess.run([sys.executable, "-c", script], capture_output=True, text=True, env=env, timeout=600)
    env["CEC_CUTS_LISTS"] = "1"
    b = subprocess.run([sys.executable, "-c", script], capture_output=True, text=True, env=env, timeout=600)
    assert a.returncode == 0 and b.returncode == 0, a.stderr[-500:] + b.stderr[-500:]
    assert a.stdout.strip() == b.stdout.strip() and len(a.stdout.strip()) == 40


def test_check_log_entries():
    """driver.CheckLog: per-pass arrays in, the replay entries (dicts) out, in issue order."""
    L = driver.CheckLog()
    assert len(L) == 0 and not L
    L.add(0, 1, 2, np.array([2, 4]), np.array([6, 9]), np.array([0, 2, 3]), np.array([1, 2, 3]), np.array([1, 0]))
    L.append({"version": 1, "phase": 2, "pass": 0, "lit_a": 10, "lit_b": 12, "leaves": [5, 6], "verdict": 1})
    assert len(L) == 3 and L
    assert L[0] == {"version": 0, "phase": 1, "pass": 2, "lit_a": 2, "lit_b": 6, "leaves": [1, 2], "verdict": 1}
    assert L[1]["leaves"] == [3] and L[1]["verdict"] == 0 and L[-1]["lit_a"] == 10
    assert [c["lit_b"] for c in L] == [6, 9, 12] and [c["lit_a"] for c in L[1:]] == [4, 10]
