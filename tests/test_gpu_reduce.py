"""GPU miter reduction (cec_reduce) against the reduction oracle
(oracle/reduce.py, P:61/:185/:187): new fanins, the image of every old node and mapped literals must
be identical, array for array. CPU part: argument checking and the no-CPU-fallback rule."""
import numpy as np
import pytest

from oracle.reduce import reduce_miter
from paper_conf_dac_liuy25_b200 import capi
from workloads import c1_add8, c3_rand, c5_big, tiny_random


def _oracle(aig, subst, lits):
    fan = [(int(a), int(b)) for a, b in aig.fanins]
    out, image, ml = reduce_miter(aig.num_pis, fan, subst, lits)
    return np.array(out, dtype=np.uint32).reshape(-1, 2), np.array(image, dtype=np.uint32), np.array(ml, dtype=np.uint32)


def _random_subst(aig, frac, rng):
    I, A = aig.num_pis, aig.num_ands
    subst = {}
    for nid in range(I + 1, I + 1 + A):
        if rng.random() < frac:
            subst[nid] = int(rng.integers(0, nid)) * 2 + int(rng.integers(0, 2))
    return subst


def _check(aig, subst, lits):
    ctx = capi.Context.from_aig(aig, device=0)
    try:
        mem = np.array(sorted(subst), dtype=np.uint32)
        rep = np.array([subst[int(m)] for m in mem], dtype=np.uint32)
        fan, img, ml = ctx.reduce(mem, rep, lits)
    finally:
        ctx.close()
    ofan, oimg, oml = _oracle(aig, subst, lits)
    assert fan.shape == ofan.shape and np.array_equal(fan, ofan)
    assert np.array_equal(img, oimg)
    assert np.array_equal(ml, oml)
    return fan


def test_reduce_bad_args_cpu():
    m = c1_add8()
    ctx = capi.Context.from_aig(m.aig, device=-1)
    I = m.aig.num_pis
    for mem, rep in (([I], [0]), ([I + 5], [2 * (I + 5)]), ([I + 5, I + 5], [0, 1]), ([10 ** 6], [0])):
        with pytest.raises(capi.CecError) as ei:
            ctx.reduce(mem, rep)
        assert ei.value.status == capi.CEC_E_ARG
    with pytest.raises(capi.CecError) as ei:  # valid merges, but no device: no CPU fallback
        ctx.reduce([I + 5], [2])
    assert ei.value.status == capi.CEC_E_CUDA
    ctx.close()


@pytest.mark.gpu
@pytest.mark.parametrize("seed", range(16))
def test_reduce_tiny_random(seed):
    m = tiny_random(num_pis=2 + seed % 9, n_ands=20 + 13 * seed, n_pairs=4, seed=300 + seed)
    rng = np.random.default_rng(seed)
    lits = list(m.lit_a) + list(m.lit_b)
    for frac in (0.0, 0.1, 0.5, 1.0):
        _check(m.aig, _random_subst(m.aig, frac, rng), lits)


@pytest.mark.gpu
def test_reduce_identity_and_po_merge_c1():
    m = c1_add8()
    fan = _check(m.aig, {}, list(m.lit_a))
    assert np.array_equal(fan, np.sort(m.aig.fanins, axis=1))
    # P phase outcome: every B-side PO merged into its A-side PO
    subst = {}
    for a, b in zip(m.lit_a, m.lit_b):
        hi, lo = (int(a), int(b)) if (a >> 1) > (b >> 1) else (int(b), int(a))
        if (hi >> 1) > m.aig.num_pis and (hi >> 1) != (lo >> 1) and (hi >> 1) not in subst:
            subst[hi >> 1] = lo ^ (hi & 1)
    _check(m.aig, subst, list(m.lit_a) + list(m.lit_b))


@pytest.mark.gpu
def test_reduce_c3_random_merges():
    m = c3_rand()
    rng = np.random.default_rng(5)
    _check(m.aig, _random_subst(m.aig, 0.02, rng), list(m.lit_a[:200]) + list(m.lit_b[:200]))


@pytest.mark.gpu
def test_reduce_c5_po_merges():
    """Full-size C5 (2.1M ANDs): every PO pair merged (the miter collapses to the A side)."""
    m = c5_big()
    subst = {}
    for a, b in zip(m.lit_a, m.lit_b):
        hi, lo = (int(a), int(b)) if (a >> 1) > (b >> 1) else (int(b), int(a))
        if (hi >> 1) > m.aig.num_pis and (hi >> 1) != (lo >> 1) and (hi >> 1) not in subst:
            subst[hi >> 1] = lo ^ (hi & 1)
    _check(m.aig, subst, list(m.lit_a) + list(m.lit_b))
