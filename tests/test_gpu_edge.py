"""Edge cases of the exhaustive check on the GPU, each against a closed form
or the oracle: no pairs, an AIG without AND nodes, constants and PIs as pair members, duplicate
pairs, and the largest enumerated window (k = 32: 2^32 patterns) with a closed-form first CEX."""
import numpy as np
import pytest

import oracle
from paper_conf_dac_liuy25_b200 import capi
from workloads import Builder, circuits

pytestmark = pytest.mark.gpu
EQ, NEQ, UND = capi.CEC_EQUIVALENT, capi.CEC_NOT_EQUIVALENT, capi.CEC_UNDECIDED


def test_no_pairs():
    bd = Builder(3)
    x = [bd.pi(i) for i in range(3)]
    aig = bd.finish([bd.AND(x[0], x[1])])
    ctx = capi.Context.from_aig(aig, device=0)
    v, c, k = ctx.sim_exhaustive([], [])
    assert v.size == 0 and c.size == 0 and k.size == 0
    ctx.close()


def test_aig_without_ands_constants_and_pis():
    bd = Builder(3)
    aig = bd.finish([bd.pi(0)])
    la = [0, 0, 2, 2, 2, 3, 6]
    lb = [0, 1, 2, 3, 4, 4, 1]
    ctx = capi.Context.from_aig(aig, device=0)
    v, c, k = ctx.sim_exhaustive(la, lb)
    # (0,0) EQ; (0,1) NEQ at 0 (k=0); x1 vs x1 EQ; x1 vs !x1 NEQ at 0; x1 vs x2: first mismatch
    # x1=1,x2=0 -> index 1; !x1 vs x2: x1=0,x2=0 -> index 0; x3 vs 1: x3=0 -> index 0
    assert list(v) == [EQ, NEQ, EQ, NEQ, NEQ, NEQ, NEQ]
    assert [int(x) for x, vv in zip(c, v) if vv == NEQ] == [0, 0, 1, 0, 0]
    assert list(k) == [0, 0, 1, 1, 2, 2, 1]
    orc = oracle.Oracle.from_aig(aig)
    ov, oc, ok, _ = orc.check_pairs(la, lb)
    assert list(ov) == list(v) and list(ok) == list(k)
    ctx.close()


def test_duplicate_pairs_identical_results():
    bd = Builder(6)
    x = [bd.pi(i) for i in range(6)]
    a = bd.AND(bd.XOR(x[0], x[1]), bd.OR(x[2], x[3]))
    b = bd.AND(bd.XOR_alt(x[0], x[1]), bd.OR(x[2], x[4]))  # differs when x3 != x4
    aig = bd.finish([a, b])
    ctx = capi.Context.from_aig(aig, device=0)
    v, c, k = ctx.sim_exhaustive([a, a, a ^ 1, a], [b, b, b ^ 1, b])
    assert list(v) == [NEQ] * 4 and len(set(int(t) for t in c)) == 1 and len(set(int(t) for t in k)) == 1
    orc = oracle.Oracle.from_aig(aig)
    ov, oc, ok, _ = orc.check_pairs([a], [b])
    assert int(oc[0]) == int(c[0]) and int(ok[0]) == int(k[0])
    ctx.close()


@pytest.mark.parametrize("engine", [capi.CEC_ENGINE_AUTO, capi.CEC_ENGINE_INTERP])
def test_k32_window_closed_form(engine):
    """32-input AND chain vs balanced AND tree (EQ), and vs the AND of the first 31 inputs (NEQ):
    they differ only when x1..x31 = 1 and x32 = 0, i.e. at own index 2^31 - 1 (P:33 convention)."""
    bd = Builder(32)
    x = [bd.pi(i) for i in range(32)]
    chain = x[0]
    for t in x[1:]:
        chain = bd.AND(chain, t)

    def tree(v):
        while len(v) > 1:
            v = [bd.AND(v[i], v[i + 1]) if i + 1 < len(v) else v[i] for i in range(0, len(v), 2)]
        return v[0]

    bal = tree(list(reversed(x)))
    part = tree(x[:31])
    aig = bd.finish([chain, bal, part])
    ctx = capi.Context.from_aig(aig, device=0, engine=engine)
    v, c, k = ctx.sim_exhaustive([chain, chain, chain], [bal, part, bal ^ 1])
    assert list(k) == [32, 32, 32]
    assert list(v) == [EQ, NEQ, NEQ]
    assert int(c[1]) == (1 << 31) - 1
    assert int(c[2]) == 0  # chain vs !bal: they differ on every pattern
    vec = ctx.get_cex(1)
    assert list(vec) == [1] * 31 + [0]
    ctx.close()


def _minterm(bd, lits, value):
    """AND of the literals of `lits` set to the bits of `value` (bit j <-> lits[j])."""
    m = 1
    for j, l in enumerate(lits):
        m = bd.AND(m, l if (value >> j) & 1 else l ^ 1)
    return m


def test_own_index_closed_form_V4_merged_windows():
    """SURVEY.md §8(c) V4 / Q8 (P:33 index convention, P:81 support order, a11 pext): an 8-bit
    ripple adder; s3 is compared with s3 XOR [a=11, b=6] (one differing pattern) and s1 with
    s1 XOR [a=3, b=2]. The closed-form own indices are 11 + 16*6 = 107 and 3 + 4*2 = 11. The two
    pairs share one merged window (supp(s1) is inside supp(s3)), so the second result must come
    back through the pext of the merged index. Also checked against the oracle."""
    bd = Builder(16)
    a = [bd.pi(i) for i in range(8)]
    b = [bd.pi(8 + i) for i in range(8)]
    s, _ = circuits.ripple_adder(bd, a, b)
    g3 = bd.XOR(s[3], _minterm(bd, a[:4] + b[:4], 11 | 6 << 4))
    g1 = bd.XOR(s[1], _minterm(bd, a[:2] + b[:2], 3 | 2 << 2))
    aig = bd.finish([s[3], g3, s[1], g1])
    la, lb = [s[3], s[1], s[3]], [g3, g1, s[3]]
    ctx = capi.Context.from_aig(aig, device=0)
    v, c, k = ctx.sim_exhaustive(la, lb)
    assert list(v) == [NEQ, NEQ, EQ]
    assert list(k) == [8, 4, 8]
    assert int(c[0]) == 107 and int(c[1]) == 11
    orc = oracle.Oracle.from_aig(aig)
    ov, oc, ok, _ = orc.check_pairs(la, lb)
    assert list(ov) == list(v) and list(ok) == list(k)
    assert [int(x) for x in oc[:2]] == [107, 11]
    ctx.close()


def test_k41_maximum_window_closed_form():
    """The largest enumerated window (k = 41 = the enumeration limit, 2^41 patterns = 2^31 JIT
    slices: the top of the u32 slice range; input 40 is bit 30 of the slice index). A 41-input AND
    chain vs a balanced tree is EQ over the whole cube; vs constant 0 it differs ONLY at the very
    last pattern, own index 2^41 - 1, so the last slice must be simulated; vs the AND of the first
    40 inputs it first differs at 2^40 - 1 (x1..x40 = 1, x41 = 0). k = 42 exceeds the limit and is
    routed to UNDECIDED even with k_max = 63. Closed forms (P:33 index convention)."""
    bd = Builder(42)
    x = [bd.pi(i) for i in range(42)]

    def chain(v):
        c = v[0]
        for t in v[1:]:
            c = bd.AND(c, t)
        return c

    def tree(v):
        while len(v) > 1:
            v = [bd.AND(v[i], v[i + 1]) if i + 1 < len(v) else v[i] for i in range(0, len(v), 2)]
        return v[0]

    c41, t41, c40, c42 = chain(x[:41]), tree(list(reversed(x[:41]))), tree(x[:40]), chain(x)
    aig = bd.finish([c41, t41, c40, c42])
    ctx = capi.Context.from_aig(aig, device=0, k_max=63, engine=capi.CEC_ENGINE_JIT)
    v, c, k = ctx.sim_exhaustive([c41, c41, c40, c42], [t41, 0, c41, 0])
    assert list(k) == [41, 41, 41, 42]
    assert list(v) == [EQ, NEQ, NEQ, UND]
    assert int(c[1]) == (1 << 41) - 1
    assert int(c[2]) == (1 << 40) - 1
    assert list(ctx.get_cex(1)) == [1] * 41 + [0]
    assert list(ctx.get_cex(2)) == [1] * 40 + [0, 0]
    ctx.close()
