"""GPU equivalence classes (cec_sim_classes) against the class oracle
(oracle/classes.py, P:41/:61/:183/:187): the (repr, member, phase) pair lists must be identical —
random patterns, caller (CEX) patterns, and both together. CPU part: argument checks and the
no-CPU-fallback rule."""
import numpy as np
import pytest

import oracle
from oracle.classes import classes
from paper_conf_dac_liuy25_b200 import capi
from workloads import c1_add8, c2_mul12_bug, c3_rand, tiny_random


def _gpu(aig, W, seed, words=None):
    ctx = capi.Context.from_aig(aig, device=0)
    try:
        r, m, ph = ctx.sim_classes(W, seed, words)
    finally:
        ctx.close()
    return [(int(a), int(b), int(c)) for a, b, c in zip(r, m, ph)]


def test_sim_classes_cpu_args():
    m = c1_add8()
    ctx = capi.Context.from_aig(m.aig, device=-1)
    with pytest.raises(capi.CecError) as ei:
        ctx.sim_classes(0, 1)  # no patterns at all
    assert ei.value.status == capi.CEC_E_ARG
    with pytest.raises(capi.CecError) as ei:
        ctx.sim_classes(4, 1)
    assert ei.value.status == capi.CEC_E_CUDA
    ctx.close()


@pytest.mark.gpu
@pytest.mark.parametrize("seed", range(12))
def test_classes_tiny_random(seed):
    m = tiny_random(num_pis=2 + seed % 10, n_ands=30 + 11 * seed, n_pairs=1, seed=700 + seed)
    orc = oracle.Oracle.from_aig(m.aig)
    rng = np.random.default_rng(seed)
    words = rng.integers(0, 1 << 32, size=(m.aig.num_pis, 1 + seed % 3), dtype=np.uint64).astype(np.uint32)
    for W, wd in ((1 + seed % 4, None), (0, words), (2, words)):
        assert _gpu(m.aig, W, seed, wd) == classes(orc, W, seed, wd), (seed, W)


@pytest.mark.gpu
@pytest.mark.parametrize("make", [c1_add8, lambda: c2_mul12_bug(seed=1)])
def test_classes_arith_miters(make):
    m = make()
    orc = oracle.Oracle.from_aig(m.aig)
    assert _gpu(m.aig, 8, 3) == classes(orc, 8, 3)


@pytest.mark.gpu
def test_classes_c3_full_size():
    """C3 (234k ANDs) at the driver's default 64 random words: identical pair list."""
    m = c3_rand()
    orc = oracle.Oracle.from_aig(m.aig)
    assert _gpu(m.aig, 64, 1) == classes(orc, 64, 1)


@pytest.mark.gpu
def test_classes_cap_truncates():
    m = c2_mul12_bug(seed=1)
    ctx = capi.Context.from_aig(m.aig, device=0)
    r, mm, ph = ctx.sim_classes(4, 3)
    r2, m2, p2 = ctx.sim_classes(4, 3, cap=5)
    ctx.close()
    assert len(r) > 5 and np.array_equal(m2, mm[:5]) and np.array_equal(r2, r[:5]) and np.array_equal(p2, ph[:5])
