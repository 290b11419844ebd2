"""Pins of the CPU oracle against things other than itself (task rule ③): the paper's worked
examples (tests/golden/paper_examples.json, each cited), arithmetic closed forms, invariants,
injected bugs and an independent pure-Python brute-force enumerator. No GPU needed."""
import json
import os

import numpy as np
import pytest

import oracle
from oracle import EQUIVALENT as EQ, NOT_EQUIVALENT as NEQ, UNDECIDED as UND, BADCUT, Oracle
from oracle import brute
from workloads import Builder, circuits, c1_add8, rewrite_copy, tiny_random

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "paper_examples.json")))


def tt_string(orc: Oracle, lit: int, ref_lit: int, k: int) -> str:
    """Truth table b_{l-1}..b_0 of `lit` over the support of (lit, ref_lit), using the oracle's own
    pattern -> assignment mapping (cex_vector) and its evaluator."""
    bits = []
    for i in range(1 << k):
        bits.append(orc.eval_lit(lit, orc.cex_vector(lit, ref_lit, i)))
    return "".join(str(b) for b in reversed(bits))


def v1_aig(order_yxz=False):
    """f = xy' + xy'z; PIs (x,y,z) = (1,2,3) or (y,x,z) = (1,2,3)."""
    bd = Builder(3, strash=False)
    x, y, z = (bd.pi(1), bd.pi(0), bd.pi(2)) if order_yxz else (bd.pi(0), bd.pi(1), bd.pi(2))
    n4 = bd.raw_and(x, y ^ 1)          # x y'
    n5 = bd.raw_and(n4, z)             # x y' z
    f = bd.raw_and(n4 ^ 1, n5 ^ 1) ^ 1  # n4 + n5
    return bd.finish([f, n4]), f, n4, x, y, z


def test_projection_truth_tables_P33():
    aig, f, n4, x, y, z = v1_aig()
    orc = Oracle.from_aig(aig)
    g = GOLD["projection_k3"]
    assert tt_string(orc, x, f, 3) == g["x0"]
    assert tt_string(orc, y, f, 3) == g["x1"]
    assert tt_string(orc, z, f, 3) == g["x2"]


def test_input_order_example_P67_P79():
    g = GOLD["xy_bar_plus_xy_bar_z"]
    aig, f, n4, x, y, z = v1_aig()
    orc = Oracle.from_aig(aig)
    assert tt_string(orc, f, f, 3) == g["order_xyz"]
    aig2, f2, *_ = v1_aig(order_yxz=True)
    orc2 = Oracle.from_aig(aig2)
    assert tt_string(orc2, f2, f2, 3) == g["order_yxz"]
    # xy' over (x, y) is 0010
    assert tt_string(orc, n4, n4, 2) == GOLD["xy_bar_two_inputs"]["order_xy"]
    # and f == xy' is a global EQ even though supp(f) = {x,y,z} != supp(xy')
    v, cex, k, _ = orc.check_pairs([f], [n4])
    assert (v[0], k[0]) == (EQ, 3)
    # f vs x: first mismatch at x=1,y=1,z=0 -> i = 0b011 = 3
    v, cex, k, _ = orc.check_pairs([f], [x])
    assert (v[0], int(cex[0]), k[0]) == (NEQ, 3, 3)


def sdc_aig():
    """n1 = x+y, n2 = yz, n3 = n1 n2 (survey vector V2)."""
    bd = Builder(3, strash=False)
    x, y, z = bd.pi(0), bd.pi(1), bd.pi(2)
    n4 = bd.raw_and(x ^ 1, y ^ 1)  # n1 = lit 9 = !n4
    n5 = bd.raw_and(y, z)          # n2 = lit 10
    n6 = bd.raw_and(n4 ^ 1, n5)    # n3 = lit 12
    return bd.finish([n6]), n4, n5, n6


def test_sdc_example_P35_P130():
    aig, n4, n5, n6 = sdc_aig()
    orc = Oracle.from_aig(aig)
    v, cex, k, _ = orc.check_pairs([n6], [n5])
    assert GOLD["sdc_example"]["global_n3_vs_n2"] == "EQ" and v[0] == EQ and k[0] == 3
    lv = orc.check_local([n6], [n5], [0, 2], [n4 >> 1, n5 >> 1])
    assert GOLD["sdc_example"]["local_n3_vs_n2_on_n1_n2"] == "UND" and lv[0] == UND
    # the cut {x,y,z} (= the support) makes the local check exact: EQ
    assert orc.check_local([n6], [n5], [0, 3], [1, 2, 3])[0] == EQ
    # {n1} alone is not a cut of n2 (y,z reachable): rejected
    assert orc.check_local([n6], [n5], [0, 1], [n4 >> 1])[0] == BADCUT


def test_special_pairs():
    aig, f, n4, x, y, z = v1_aig()
    orc = Oracle.from_aig(aig)
    v, cex, k, _ = orc.check_pairs([0, f, f, 0], [1, f, f ^ 1, 0])
    assert list(v) == [NEQ, EQ, NEQ, EQ]
    assert int(cex[0]) == 0 and k[0] == 0          # V5: (0, 1) -> NEQ at index 0, k = 0
    assert int(cex[2]) == 0                          # antivalent literals differ everywhere
    assert list(orc.cex_vector(0, 1, 0)) == [0, 0, 0]
    # k_max: a pair above the limit is UNDECIDED
    v, cex, k, _ = orc.check_pairs([f], [n4], k_max=2)
    assert v[0] == UND and int(cex[0]) == oracle.NO_CEX


def test_adder_closed_form_C1():
    m = c1_add8()
    orc = Oracle.from_aig(m.aig)
    rng = np.random.default_rng(0)
    for _ in range(300):
        a, b = int(rng.integers(0, 256)), int(rng.integers(0, 256))
        pis = np.array([(a >> i) & 1 for i in range(8)] + [(b >> i) & 1 for i in range(8)], dtype=np.uint8)
        s = a + b
        for j in range(9):
            assert orc.eval_lit(int(m.lit_a[j]), pis) == (s >> j) & 1
            assert orc.eval_lit(int(m.lit_b[j]), pis) == (s >> j) & 1
    v, cex, k, ev = orc.check_pairs(m.lit_a, m.lit_b)
    assert list(v) == [EQ] * 9
    assert list(k) == [2 * (j + 1) for j in range(8)] + [16]  # supp(s_i) = {a_0..a_i, b_0..b_i}


@pytest.mark.parametrize("n", [4, 6])
def test_multiplier_closed_form_and_brute(n):
    m = circuits.c2_mul12(n)
    orc = Oracle.from_aig(m.aig)
    for a in range(1 << n):
        for b in range(0, 1 << n, 3):
            pis = np.array([(a >> i) & 1 for i in range(n)] + [(b >> i) & 1 for i in range(n)], dtype=np.uint8)
            p = a * b
            j = (a + b) % (2 * n)
            assert orc.eval_lit(int(m.lit_a[j]), pis) == (p >> j) & 1
            assert orc.eval_lit(int(m.lit_b[j]), pis) == (p >> j) & 1
    v, cex, k, _ = orc.check_pairs(m.lit_a, m.lit_b)
    assert list(v) == [EQ] * (2 * n)
    if n <= 6:
        ref = brute.check_pairs(m.aig.num_pis, m.aig.fanins, list(zip(m.lit_a, m.lit_b)))
        assert [r[1] for r in ref] == list(v) and [r[0] for r in ref] == list(k)


def test_mul_bug_refuted_with_closed_form_cex():
    n = 6
    m = circuits.c2_mul12_bug(seed=1, n=n)
    orc = Oracle.from_aig(m.aig)
    v, cex, k, _ = orc.check_pairs(m.lit_a, m.lit_b)
    assert NEQ in list(v), "the injected bug must be observable and refuted"
    for j in np.nonzero(v == NEQ)[0]:
        vec = orc.cex_vector(int(m.lit_a[j]), int(m.lit_b[j]), int(cex[j]))
        a = sum(int(vec[i]) << i for i in range(n))
        b = sum(int(vec[n + i]) << i for i in range(n))
        # A side is the correct product (closed form); the buggy B side differs there
        assert orc.eval_lit(int(m.lit_a[j]), vec) == ((a * b) >> j) & 1
        assert orc.eval_lit(int(m.lit_b[j]), vec) != ((a * b) >> j) & 1
    ref = brute.check_pairs(m.aig.num_pis, m.aig.fanins, list(zip(m.lit_a, m.lit_b)))
    assert [r[1] for r in ref] == list(v)
    assert [r[2] if r[2] is not None else oracle.NO_CEX for r in ref] == [int(c) for c in cex]


@pytest.mark.parametrize("seed", range(40))
def test_brute_force_random(seed):
    rng = np.random.default_rng(seed)
    I = int(rng.integers(1, 11))
    m = tiny_random(I, int(rng.integers(1, 40)), 12, seed)
    orc = Oracle.from_aig(m.aig)
    kmax = int(rng.integers(0, 12))
    v, cex, k, _ = orc.check_pairs(m.lit_a, m.lit_b, k_max=kmax)
    ref = brute.check_pairs(I, m.aig.fanins, list(zip(m.lit_a, m.lit_b)), k_max=kmax)
    for p, (rk, rv, rc) in enumerate(ref):
        assert k[p] == rk and v[p] == rv
        assert int(cex[p]) == (rc if rc is not None else oracle.NO_CEX)


@pytest.mark.parametrize("seed", range(25))
def test_brute_force_local(seed):
    rng = np.random.default_rng(100 + seed)
    I = int(rng.integers(2, 9))
    m = tiny_random(I, int(rng.integers(3, 30)), 6, 100 + seed)
    orc = Oracle.from_aig(m.aig)
    N = m.aig.num_nodes
    la, lb, off, lv = [], [], [0], []
    for q in range(m.num_pairs):
        cand = rng.choice(np.arange(1, N), size=int(rng.integers(1, min(N - 1, 7) + 1)), replace=False)
        if rng.random() < 0.5:  # make it a valid cut: add all PIs
            cand = np.unique(np.concatenate([cand, np.arange(1, I + 1)]))
        la.append(int(m.lit_a[q])); lb.append(int(m.lit_b[q]))
        lv += [int(x) for x in cand]
        off.append(len(lv))
    got = orc.check_local(la, lb, off, lv)
    gv, gcex, gk, _ = orc.check_pairs(la, lb, k_max=63)
    for q in range(len(la)):
        want = brute.check_local(I, m.aig.fanins, la[q], lb[q], lv[off[q]:off[q + 1]])
        assert got[q] == (BADCUT if want == "BADCUT" else want)
        if got[q] == EQ:  # soundness of local checking: local EQ => global EQ
            assert gv[q] == EQ


def test_invariants_self_and_rewrite():
    for seed in range(6):
        m = circuits.random_miter(10, 200, 8, seed=seed, window=24)  # A vs rewrite_copy(A)
        orc = Oracle.from_aig(m.aig)
        v, _, _, _ = orc.check_pairs(m.lit_a, m.lit_b)
        assert list(v) == [EQ] * m.num_pairs
        v, _, _, _ = orc.check_pairs(m.lit_a, m.lit_a)
        assert list(v) == [EQ] * m.num_pairs
        ref = brute.check_pairs(10, m.aig.fanins, list(zip(m.lit_a, m.lit_b)))
        assert all(r[1] == brute.EQ for r in ref)


def test_injected_bugs_refuted():
    hits = 0
    for seed in range(8):
        m = circuits.random_miter(9, 120, 6, seed=50 + seed, window=20)
        rng = np.random.default_rng(seed)
        drv = int(m.lit_b[int(rng.integers(0, m.num_pairs))]) >> 1  # B-side AND driving a PO
        bug = circuits.flip_fanin(m, drv, int(rng.integers(0, 2)))
        orc = Oracle.from_aig(bug.aig)
        v, cex, k, _ = orc.check_pairs(bug.lit_a, bug.lit_b)
        ref = brute.check_pairs(9, bug.aig.fanins, list(zip(bug.lit_a, bug.lit_b)))
        assert [r[1] for r in ref] == list(v)
        assert [r[2] if r[2] is not None else oracle.NO_CEX for r in ref] == [int(c) for c in cex]
        hits += int(NEQ in list(v))
    assert hits >= 4


def test_range_sharding_equals_full_scan():
    """SURVEY.md §8(c) 'Sharded oracle': min over shards of first mismatch = first mismatch."""
    m = circuits.c2_mul12_bug(seed=1, n=6)
    orc = Oracle.from_aig(m.aig)
    v, cex, k, _ = orc.check_pairs(m.lit_a, m.lit_b)
    best = np.full(m.num_pairs, oracle.NO_CEX, dtype=np.uint64)
    for lo in range(0, 1 << 12, 1000):
        vs, cs, _, _ = orc.check_pairs(m.lit_a, m.lit_b, lo=lo, hi=lo + 1000)
        best = np.minimum(best, np.where(vs == NEQ, cs, oracle.NO_CEX).astype(np.uint64))
    assert [int(x) for x in best] == [int(c) if vv == NEQ else oracle.NO_CEX for vv, c in zip(v, cex)]


def test_cli_diffable_output(tmp_path):
    from workloads import write_aag, write_pairs
    m = circuits.c2_mul12_bug(seed=1, n=4)
    write_aag(m.aig, str(tmp_path / "m.aag"))
    write_pairs(str(tmp_path / "p.txt"), m.lit_a, m.lit_b)
    out = oracle.run_cli("check", str(tmp_path / "m.aag"), str(tmp_path / "p.txt")).splitlines()
    orc = Oracle.from_aig(m.aig)
    v, cex, k, _ = orc.check_pairs(m.lit_a, m.lit_b)
    names = {EQ: "EQ", NEQ: "NEQ", UND: "UND"}
    for p in range(m.num_pairs):
        f = out[p].split()
        assert f == [str(p), str(m.lit_a[p]), str(m.lit_b[p]), str(k[p]), names[v[p]],
                     str(int(cex[p])) if v[p] == NEQ else "-"]
    assert sum(1 for l in out if l.startswith("cex ")) == int((v == NEQ).sum())


def test_aiger_reader_renumbers_non_topological(tmp_path):
    # gates listed out of order: 10 = 8 & 2 before 8 = 2 & 4
    p = tmp_path / "x.aag"
    p.write_text("aag 5 3 0 1 2\n2\n4\n6\n10\n10 8 6\n8 2 4\n")
    orc = Oracle(str(p))
    assert orc.num_pis == 3 and orc.num_ands == 2
    v, cex, k, _ = orc.check_pairs([2 * 5], [2 * 5])
    assert v[0] == EQ and k[0] == 3


def test_own_index_mapping_V4():
    """SURVEY.md §8(c) V4 (P:33 index convention, P:81 increasing-id support order): C1 PO s3 has
    support {a0..a3, b0..b3}; the pattern a = 11, b = 6 is own index 11 + 16*6 = 107, and every
    index i of that support maps to a = i mod 16, b = i div 16 (closed form, not the oracle's
    own evaluator)."""
    m = c1_add8()
    orc = Oracle.from_aig(m.aig)
    s3a, s3b = int(m.lit_a[3]), int(m.lit_b[3])
    for i in (107, 0, 255, 16, 15):
        pis = np.asarray(orc.cex_vector(s3a, s3b, i))
        a = sum(int(pis[j]) << j for j in range(8))
        b = sum(int(pis[8 + j]) << j for j in range(8))
        assert (a & 15, b & 15) == (i % 16, i // 16)
        assert a >> 4 == 0 and b >> 4 == 0          # PIs outside the support stay 0
        assert orc.eval_lit(s3a, pis) == ((a + b) >> 3) & 1
    pis = np.asarray(orc.cex_vector(s3a, s3b, 107))
    assert [int(pis[j]) for j in range(4)] == [1, 1, 0, 1] and [int(pis[8 + j]) for j in range(4)] == [0, 1, 1, 0]


@pytest.mark.parametrize("n", [8, 64])
def test_datapath_closed_form_C4(n):
    """C4: both sides of the n-bit datapath miter compute s = a + b + cin,
    lt = (a < b) and y = lt ? b : a — checked bit by bit through the oracle's own evaluator at
    random assignments (arithmetic, not the oracle, is the reference), and the bug variant's B side
    differs from the closed form at some assignment the oracle finds (it must never be EQ)."""
    m = circuits.c4_dp(n)
    orc = Oracle.from_aig(m.aig)
    rng = np.random.default_rng(n)
    mask = (1 << n) - 1
    for _ in range(40):
        a = int(rng.integers(0, 1 << 62)) & mask if n > 62 else int(rng.integers(0, 1 << n))
        b = int(rng.integers(0, 1 << 62)) & mask if n > 62 else int(rng.integers(0, 1 << n))
        if n > 62:
            a |= int(rng.integers(0, 4)) << 62
            b |= int(rng.integers(0, 4)) << 62
        cin = int(rng.integers(0, 2))
        pis = np.array([(a >> i) & 1 for i in range(n)] + [(b >> i) & 1 for i in range(n)] + [cin], np.uint8)
        s = a + b + cin
        want = [(s >> i) & 1 for i in range(n + 1)] + [int(a < b)] + [((b if a < b else a) >> i) & 1 for i in range(n)]
        for side in (m.lit_a, m.lit_b):
            got = [orc.eval_lit(int(l), pis) for l in side]
            assert got == want, (n, a, b, cin)
    if n == 8:  # small enough for the exhaustive oracle: the bug variant is refuted, never EQ
        mb = circuits.c4_dp(n, bug=4)
        ob = Oracle.from_aig(mb.aig)
        v, _, _, _ = ob.check_pairs(mb.lit_a, mb.lit_b, k_max=17)
        assert (v == NEQ).any() and not (v == EQ).all()
