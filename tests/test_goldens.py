"""CPU checks of the stored full-size oracle results (tests/golden/*.json, written by
scripts/make_golden*.py, which call only oracle/): they still describe the miters the seeded
generators build today, and every stored counter-example is re-checked by the oracle's single-
assignment evaluator — a path independent of the enumeration loop that produced it (a separating
assignment must make the two literals differ, SURVEY.md §8(c) "CEX vector")."""
import json
import os

import numpy as np
import pytest

import oracle
from workloads import c1_add8, c2_mul12, c2_mul12_bug, c3_rand, c5_big

GOLD = os.path.join(os.path.dirname(__file__), "golden")
CASES = {
    "c1_add8": lambda: c1_add8(),
    "c2_mul12": lambda: c2_mul12(),
    "c2_mul12_bug1": lambda: c2_mul12_bug(seed=1),
    "c3_rand": lambda: c3_rand(),
    "c5_big": lambda: c5_big(),
}


@pytest.mark.parametrize("name", sorted(CASES))
def test_golden_matches_generator_and_cex_separates(name):
    path = os.path.join(GOLD, name + ".json")
    if not os.path.exists(path):
        pytest.skip(f"{path} missing")
    g = json.load(open(path))
    m = CASES[name]()
    assert g["num_pis"] == m.aig.num_pis and g["num_ands"] == m.aig.num_ands
    assert g["lit_a"] == [int(x) for x in m.lit_a] and g["lit_b"] == [int(x) for x in m.lit_b]
    v = np.array(g["verdict"])
    assert set(np.unique(v)) <= {oracle.EQUIVALENT, oracle.NOT_EQUIVALENT}  # every k <= 32 here
    orc = oracle.Oracle.from_aig(m.aig)
    neq = np.nonzero(v == oracle.NOT_EQUIVALENT)[0]
    for p in neq:
        la, lb, idx = int(m.lit_a[p]), int(m.lit_b[p]), int(g["cex"][p])
        assert idx < (1 << int(g["k"][p]))
        vec = orc.cex_vector(la, lb, idx)
        assert orc.eval_lit(la, vec) != orc.eval_lit(lb, vec), (name, p, idx)
    # the bug-free configurations have no NEQ pair; the bugged ones do
    assert (len(neq) == 0) == (name in ("c1_add8", "c2_mul12"))
    if name == "c5_big":
        assert len(neq) == 8  # one observable bug per bugged copy
