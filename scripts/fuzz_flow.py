"""Fuzz campaign (GPU) of the whole P -> G -> L* flow (driver.check_miter, §III-D) against
the oracle: random-block miters A vs a rewritten A (10..14 PIs, so every PO is also checkable
exhaustively), a third of them with an injected single-gate bug. Per miter: every PO the flow
decides must agree with the oracle's exhaustive PO verdict (EQ only where the oracle says EQ, NEQ
only where it says NEQ; with these thresholds POs of support > k_P may stay UNDECIDED),
a NEQ verdict's CEX must separate the POs under the oracle's evaluator, and every logged local check
is replayed through the oracle on the miter version it ran on (bit-exact verdicts). The small
thresholds (k_P = k_p = k_g = 6, k_l = 8, C = 8) force local phases. One JSON line with the counts
and any failing seed (none expected).

  python scripts/fuzz_flow.py [--seeds 100] [--start 0]
"""
import argparse
import json
import os
import sys
import time
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import oracle  # noqa: E402
from paper_conf_dac_liuy25_b200 import capi, driver  # noqa: E402
from workloads import circuits  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--seeds", type=int, default=100)
    ap.add_argument("--start", type=int, default=0)
    a = ap.parse_args()
    p = driver.CecParams(k_P=6, k_p=6, k_g=6, k_l=8, C=8)
    bad, pos, neq, checks, local_eq, und, eqd, t0 = [], 0, 0, 0, 0, 0, 0, time.time()
    for seed in range(a.start, a.start + a.seeds):
        rng = np.random.default_rng(123000 + seed)
        I = int(rng.integers(10, 15))
        m = circuits.random_miter(I, int(rng.integers(120, 500)), 8, seed=124000 + seed,
                                  window=int(rng.integers(12, 40)))
        if rng.random() < 0.33:
            lo, hi = circuits.b_side_ids(m)
            if hi > lo:
                m = circuits.flip_fanin(m, int(rng.integers(lo, hi)), int(rng.integers(0, 2)))
        res = driver.check_miter(m.aig, m.lit_a, m.lit_b, p)
        orc = oracle.Oracle.from_aig(m.aig)
        ov, oc, ok, _ = orc.check_pairs(m.lit_a, m.lit_b, k_max=32)
        good = all(int(g) == capi.CEC_UNDECIDED or int(g) == int(o) for g, o in zip(res.po_verdicts, ov))
        und += int((res.po_verdicts == capi.CEC_UNDECIDED).sum())
        eqd += int((res.po_verdicts == capi.CEC_EQUIVALENT).sum())
        if good and res.verdict == capi.CEC_NOT_EQUIVALENT:
            q = res.cex_pair
            good = orc.eval_lit(int(m.lit_a[q]), res.cex) != orc.eval_lit(int(m.lit_b[q]), res.cex)
        byv = defaultdict(list)
        for ch in res.checks:
            byv[ch["version"]].append(ch)
        for vi, chs in byv.items():
            vo = oracle.Oracle.from_aig(res.versions[vi])
            off = np.cumsum([0] + [len(c["leaves"]) for c in chs])
            want = vo.check_local([c["lit_a"] for c in chs], [c["lit_b"] for c in chs], off,
                                  [x for c in chs for x in c["leaves"]])
            good = good and [c["verdict"] for c in chs] == [int(w) for w in want]
            local_eq += sum(1 for c in chs if c["verdict"] == capi.CEC_EQUIVALENT)
        checks += len(res.checks)
        pos += m.num_pairs
        neq += int((ov == oracle.NOT_EQUIVALENT).sum())
        if not good:
            bad.append(seed)
    print(json.dumps({"fuzz": "P->G->L* flow vs oracle (PO verdicts, CEX, every local check replayed)",
                      "seeds": a.seeds, "start": a.start, "po_pairs": pos, "neq_pos": neq, "local_checks": checks,
                      "local_eq": local_eq, "po_eq_by_flow": eqd, "po_undecided": und,
                      "failing_seeds": bad, "ok": not bad,
                      "seconds": round(time.time() - t0, 1)}), flush=True)
    driver.release_contexts()
    return 1 if bad else 0


if __name__ == "__main__":
    sys.exit(main())
