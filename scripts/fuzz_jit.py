"""Fuzz campaign (GPU): the JIT engine (dual-pipe cells, free-warp and bundle kernels) against the
oracle on many seeded random AIGs with 10..16 PIs — the window sizes where inputs switch from
per-bit to lane- to slice-uniform words and IMAD cells appear. One JSON line per run with the seed
count and every mismatching seed (none expected). Evidence beyond the pytest suite's fixed seeds.

  python scripts/fuzz_jit.py [--seeds 300] [--start 0]
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import oracle  # noqa: E402
from paper_conf_dac_liuy25_b200 import capi  # noqa: E402
from workloads import circuits, tiny_random  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--seeds", type=int, default=300)
    ap.add_argument("--start", type=int, default=0)
    ap.add_argument("--engine", default="jit", choices=["jit", "auto", "interp"],
                    help="engine under test (auto: per-window JIT / interpreter choice, as the product runs)")
    ap.add_argument("--split", type=float, default=-1.0,
                    help="CEC_PIPE_SPLIT for the public call (with CEC_PIPE_SPLIT_MINWIN=2): large windows first")
    ap.add_argument("--miters", action="store_true",
                    help="random-block miters A vs rewritten A (mostly EQ: full sweeps) instead of random pairs")
    a = ap.parse_args()
    engine = {"jit": capi.CEC_ENGINE_JIT, "auto": capi.CEC_ENGINE_AUTO, "interp": capi.CEC_ENGINE_INTERP}[a.engine]
    if a.split >= 0:
        os.environ["CEC_PIPE_SPLIT"] = str(a.split)
        os.environ["CEC_PIPE_SPLIT_MINWIN"] = "2"
    bad, pairs, neq, t0 = [], 0, 0, time.time()
    for seed in range(a.start, a.start + a.seeds):
        rng = np.random.default_rng(70000 + seed)
        I = int(rng.integers(10, 17))
        if a.miters:
            m = circuits.random_miter(I, int(rng.integers(100, 600)), 12, seed=90000 + seed,
                                      window=int(rng.integers(16, 64)))
            if rng.random() < 0.3:  # an injected observable-or-not single-gate bug in B
                lo, hi = circuits.b_side_ids(m)
                if hi > lo:
                    m = circuits.flip_fanin(m, int(rng.integers(lo, hi)), int(rng.integers(0, 2)))
        else:
            m = tiny_random(I, int(rng.integers(30, 400)), 24, 80000 + seed)
        merge = int(rng.integers(0, 3))
        ctx = capi.Context.from_aig(m.aig, k_max=16, merge=merge, engine=engine)
        gv, gc, gk = ctx.sim_exhaustive(m.lit_a, m.lit_b)
        orc = oracle.Oracle.from_aig(m.aig)
        ov, oc, ok, _ = orc.check_pairs(m.lit_a, m.lit_b, k_max=16)
        same = list(map(int, gv)) == list(map(int, ov)) and list(map(int, gk)) == list(map(int, ok))
        for p in range(m.num_pairs):
            if same and int(gv[p]) == oracle.NOT_EQUIVALENT:
                same = int(gc[p]) == int(oc[p])
                if same:
                    vec = ctx.get_cex(p)
                    same = bool(np.array_equal(vec, orc.cex_vector(int(m.lit_a[p]), int(m.lit_b[p]), int(oc[p]))))
        if not same:
            bad.append(seed)
        pairs += m.num_pairs
        neq += int((ov == oracle.NOT_EQUIVALENT).sum())
        ctx.close()
    print(json.dumps({"fuzz": f"{a.engine} engine vs oracle" + (" (A vs rewritten A miters)" if a.miters else "")
                      + (f", split {a.split}" if a.split >= 0 else ""), "seeds": a.seeds, "start": a.start, "pairs": pairs,
                      "neq_pairs": neq, "mismatching_seeds": bad, "ok": not bad,
                      "seconds": round(time.time() - t0, 1)}), flush=True)
    return 1 if bad else 0


if __name__ == "__main__":
    sys.exit(main())
