"""Write oracle results for the full-size configs C1, C2 and C2-bug (C2's oracle run takes minutes).

Calls only oracle/ (and the seeded generators). Output: tests/golden/<name>.json with per-pair
verdict, k and canonical CEX index, plus the generator parameters, so GPU parity tests on the box
compare against stored oracle values instead of re-running a multi-minute CPU scan."""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
from workloads import c1_add8, c2_mul12, c2_mul12_bug  # noqa: E402

CASES = {
    "c1_add8": (c1_add8, {}),
    "c2_mul12": (c2_mul12, {}),
    "c2_mul12_bug1": (c2_mul12_bug, {"seed": 1}),
}


def main(names):
    for name in names:
        fn, kw = CASES[name]
        m = fn(**kw)
        orc = oracle.Oracle.from_aig(m.aig)
        t = time.time()
        v, cex, k, ev = orc.check_pairs(m.lit_a, m.lit_b, k_max=32)
        dt = time.time() - t
        out = {
            "_about": f"oracle/ results for workloads.{fn.__name__}(**{kw}); written by scripts/make_golden.py",
            "generator": fn.__name__, "kwargs": kw,
            "num_pis": int(m.aig.num_pis), "num_ands": int(m.aig.num_ands),
            "lit_a": [int(x) for x in m.lit_a], "lit_b": [int(x) for x in m.lit_b],
            "verdict": [int(x) for x in v], "k": [int(x) for x in k],
            "cex": [int(x) for x in cex],
            "oracle_node_evals": int(ev), "oracle_seconds": round(dt, 2),
        }
        path = os.path.join(ROOT, "tests", "golden", name + ".json")
        with open(path, "w") as fh:
            json.dump(out, fh, indent=1)
        print(name, dt, "s", file=sys.stderr)


if __name__ == "__main__":
    main(sys.argv[1:] or list(CASES))
