"""Write the oracle's result for EVERY pair of the full-size C5 miter (workloads.c5_big()):
tests/golden/c5_big.json with per-pair verdict, k and canonical CEX index.

Calls only oracle/ (and the seeded generators). Each of the 256 copies is one task: its PO pairs are
checked by the single-threaded oracle over the full 2^24-pattern space (one assignment at a time);
tasks run in independent processes (the "sharded oracle" of SURVEY.md §8(c): pair-only sharding,
no reduction needed). About 6 core-hours. Usage: nice python scripts/make_golden_c5.py [procs]"""
import json
import multiprocessing as mp
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

_m = None
_orc = None


def _init():
    global _m, _orc
    import oracle
    from workloads import c5_big
    _m = c5_big()
    _orc = oracle.Oracle.from_aig(_m.aig)


def _copy(c):
    ppc = _m.meta["pairs_per_copy"]
    off = int(np.sum(ppc[:c]))
    n = int(ppc[c])
    t = time.time()
    v, cex, k, ev = _orc.check_pairs(_m.lit_a[off:off + n], _m.lit_b[off:off + n], k_max=32)
    return c, off, [int(x) for x in v], [int(x) for x in cex], [int(x) for x in k], int(ev), time.time() - t


def main():
    procs = int(sys.argv[1]) if len(sys.argv) > 1 else max(1, os.cpu_count() - 1)
    # optional copy range [lo, hi) (several hosts can work on disjoint ranges; their partial files
    # are concatenated afterwards) and partial-file path (GOLDEN_PARTIAL)
    lo = int(sys.argv[2]) if len(sys.argv) > 2 else 0
    hi = int(sys.argv[3]) if len(sys.argv) > 3 else 1 << 30
    from workloads import c5_big
    m = c5_big()
    P = m.num_pairs
    ncopy = len(m.meta["pairs_per_copy"])
    V, X, K = [None] * P, [None] * P, [None] * P
    evals, cpu_s = 0, 0.0
    t0 = time.time()
    # per-copy checkpoint (resumable: a restarted run skips the copies already in it)
    part = os.environ.get("GOLDEN_PARTIAL", os.path.join(ROOT, "tests", "golden", "c5_big.partial.jsonl"))
    done = set()
    if os.path.exists(part):
        with open(part) as fh:
            for line in fh:
                if not line.strip():
                    continue
                r = json.loads(line)
                c, off, v, cex, k = r["copy"], r["off"], r["v"], r["cex"], r["k"]
                V[off:off + len(v)], X[off:off + len(v)], K[off:off + len(v)] = v, cex, k
                evals += r["ev"]
                cpu_s += r["dt"]
                done.add(c)
    todo = [c for c in range(max(0, lo), min(ncopy, hi)) if c not in done]
    with mp.Pool(procs, initializer=_init) as pool, open(part, "a") as pf:
        for i, (c, off, v, cex, k, ev, dt) in enumerate(pool.imap_unordered(_copy, todo)):
            V[off:off + len(v)], X[off:off + len(v)], K[off:off + len(v)] = v, cex, k
            evals += ev
            cpu_s += dt
            pf.write(json.dumps({"copy": c, "off": off, "v": v, "cex": cex, "k": k,
                                 "ev": ev, "dt": round(dt, 2)}) + "\n")
            pf.flush()
            print(f"copy {c} done ({len(done) + i + 1}/{ncopy}) {dt:.1f}s", file=sys.stderr, flush=True)
    if any(v is None for v in V):
        print(f"partial: copies [{lo}, {hi}) done into {part}", file=sys.stderr)
        return
    out = {
        "_about": "oracle/ results for every pair of workloads.c5_big() (defaults); written by "
                  "scripts/make_golden_c5.py (one single-threaded oracle task per copy)",
        "generator": "c5_big", "kwargs": {},
        "num_pis": int(m.aig.num_pis), "num_ands": int(m.aig.num_ands),
        "lit_a": [int(x) for x in m.lit_a], "lit_b": [int(x) for x in m.lit_b],
        "verdict": V, "k": K, "cex": X,
        "oracle_node_evals": evals, "oracle_cpu_seconds": round(cpu_s, 1),
        "oracle_wall_seconds": round(time.time() - t0, 1), "oracle_processes": procs,
    }
    with open(os.path.join(ROOT, "tests", "golden", "c5_big.json"), "w") as fh:
        json.dump(out, fh)
    os.remove(part)


if __name__ == "__main__":
    main()
