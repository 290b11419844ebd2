"""Alg. 2 pass (cec_local_pass): level-by-level cut
enumeration with a common-cut buffer flushed to the local-check kernels. Its checks must be exactly
the common cuts of cec_common_cuts, each check's verdict must equal the oracle's local check
(P:128-130), pair verdicts must be "any cut proves it", and nothing may depend on the buffer size."""
import numpy as np
import pytest

import oracle
from paper_conf_dac_liuy25_b200 import capi
from workloads import c4_dp


def _pairs(m, ctx):
    r, mm, ph = ctx.sim_classes(8, 5)
    return r, mm, ph


def test_local_pass_cpu_args():
    m = c4_dp(8)
    ctx = capi.Context.from_aig(m.aig, device=-1)
    I = m.aig.num_pis
    with pytest.raises(capi.CecError) as ei:
        capi.cec_local_pass(ctx.handle, [I + 3], [I + 2], [0], 8, 8, 0, 4)  # repr >= member
    assert ei.value.status == capi.CEC_E_ARG
    with pytest.raises(capi.CecError) as ei:
        capi.cec_local_pass(ctx.handle, [I + 2], [I + 3], [0], 8, 8, 0, 4)
    assert ei.value.status == capi.CEC_E_CUDA
    ctx.close()


@pytest.mark.gpu
@pytest.mark.parametrize("n,pass_id", [(8, 0), (8, 1), (8, 2), (16, 1)])
def test_local_pass_matches_cuts_then_checks_and_oracle(n, pass_id):
    m = c4_dp(n)
    ctx = capi.Context.from_aig(m.aig, device=0, k_max=16)
    r, mm, ph = _pairs(m, ctx)
    assert r.size > 10
    k_l, C, maxc = 12, 8, 6
    # reference: the two-step route
    pco, co, lv = capi.cec_common_cuts(ctx.handle, r, mm, k_l, C, pass_id, maxc)
    la, lb, off, leaves, who = [], [], [0], [], []
    for q in range(r.size):
        for t in range(int(pco[q]), int(pco[q + 1])):
            la.append(2 * int(r[q]))
            lb.append(2 * int(mm[q]) ^ int(ph[q]))
            leaves += [int(x) for x in lv[co[t]:co[t + 1]]]
            off.append(len(leaves))
            who.append(q)
    ref_v = ctx.check_local_cuts(la, lb, off, leaves)
    ref_checks = sorted((who[i], tuple(leaves[off[i]:off[i + 1]]), int(ref_v[i])) for i in range(len(who)))
    ref_pair = np.full(r.size, capi.CEC_UNDECIDED, np.int32)
    for i, q in enumerate(who):
        if ref_v[i] == capi.CEC_EQUIVALENT:
            ref_pair[q] = capi.CEC_EQUIVALENT
    orc = oracle.Oracle.from_aig(m.aig)
    for buf in (1, 7, 4096):
        v, (cp, cof, cl, cv) = capi.cec_local_pass(ctx.handle, r, mm, ph, k_l, C, pass_id, maxc, buffer_checks=buf)
        got = sorted((int(cp[i]), tuple(int(x) for x in cl[cof[i]:cof[i + 1]]), int(cv[i])) for i in range(cp.size))
        assert got == ref_checks, buf
        assert np.array_equal(v, ref_pair), buf
    # every check's verdict is the oracle's local check
    la2 = [2 * int(r[q]) for q in cp]
    lb2 = [2 * int(mm[q]) ^ int(ph[q]) for q in cp]
    want = orc.check_local(la2, lb2, cof, cl)
    assert np.array_equal(np.asarray(cv), np.asarray(want))
    ctx.close()
