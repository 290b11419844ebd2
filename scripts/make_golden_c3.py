"""Write the oracle's result for EVERY pair of the full-size C3 miter (workloads.c3_rand()):
tests/golden/c3_rand.json with per-pair verdict, k and canonical CEX index.

Calls only oracle/ (and the seeded generators). This is SURVEY.md §8(c)'s "sharded oracle": pairs are
grouped by identical support S (the oracle shares one enumeration per group, §8(c) step 5) and a
group whose scan is long is cut into contiguous pattern-index ranges [lo, hi); every task is the
same single-threaded oracle over its range, and a pair's result is the minimum first-mismatch index
over the ranges (min over a partition of an ascending scan = first mismatch of the full scan).
About 3.6e12 node evaluations (~0.7 core-hours). Usage: nice python scripts/make_golden_c3.py [procs]"""
import collections
import json
import multiprocessing as mp
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

NO_CEX = (1 << 64) - 1
TASK_EVALS = 2e10  # ~15 s of oracle time per task
_m = None
_orc = None


def _init():
    global _m, _orc
    import oracle
    from workloads import c3_rand
    _m = c3_rand()
    _orc = oracle.Oracle.from_aig(_m.aig)


def _task(t):
    pairs, lo, hi = t
    la = [int(_m.lit_a[p]) for p in pairs]
    lb = [int(_m.lit_b[p]) for p in pairs]
    t0 = time.time()
    v, cex, k, ev = _orc.check_pairs(la, lb, k_max=32, lo=lo, hi=hi)
    return pairs, [int(x) for x in v], [int(x) for x in cex], [int(x) for x in k], int(ev), time.time() - t0


def _cone_size(f, I, roots):
    seen, st = set(), [r for r in roots if r > I]
    while st:
        v = st.pop()
        if v in seen:
            continue
        seen.add(v)
        for lit in f[v - I - 1]:
            u = int(lit) >> 1
            if u > I and u not in seen:
                st.append(u)
    return len(seen)


def main():
    procs = int(sys.argv[1]) if len(sys.argv) > 1 else max(1, os.cpu_count() - 1)
    import oracle
    from workloads import c3_rand
    m = c3_rand()
    orc = oracle.Oracle.from_aig(m.aig)
    groups = collections.defaultdict(list)
    for p, (a, b) in enumerate(zip(m.lit_a, m.lit_b)):
        groups[tuple(orc.support(int(a), int(b)))].append(p)
    f = np.asarray(m.aig.fanins).reshape(-1, 2)
    tasks = []
    for S, ps in groups.items():
        k = len(S)
        if k > 32:
            tasks.append((ps, 0, NO_CEX))  # UNDECIDED, no scan
            continue
        roots = {int(m.lit_a[p]) >> 1 for p in ps} | {int(m.lit_b[p]) >> 1 for p in ps}
        cost = (1 << k) * max(1, _cone_size(f, m.aig.num_pis, roots))
        parts = max(1, int(cost // TASK_EVALS))
        n = 1 << k
        for i in range(parts):
            tasks.append((ps, n * i // parts, n * (i + 1) // parts))
    tasks.sort(key=lambda t: -(t[2] - t[1]) if t[2] != NO_CEX else 0)
    P = m.num_pairs
    K, R = [None] * P, [[] for _ in range(P)]  # per pair: (verdict, cex) of every range
    evals, cpu_s, t0 = 0, 0.0, time.time()
    with mp.Pool(procs, initializer=_init) as pool:
        for i, (pairs, v, cex, k, ev, dt) in enumerate(pool.imap_unordered(_task, tasks)):
            for p, vv, cc, kk in zip(pairs, v, cex, k):
                K[p] = kk
                R[p].append((vv, cc))
            evals += ev
            cpu_s += dt
            if (i + 1) % 200 == 0:
                print(f"{i + 1}/{len(tasks)} tasks, {time.time() - t0:.0f} s", file=sys.stderr, flush=True)
    # NEQ if any range holds a mismatch (CEX = the minimum index), EQ if every range is clean
    V, X = [None] * P, [NO_CEX] * P
    for p in range(P):
        neq = [c for v, c in R[p] if v == oracle.NOT_EQUIVALENT]
        if neq:
            V[p], X[p] = oracle.NOT_EQUIVALENT, min(neq)
        elif R[p] and all(v == oracle.EQUIVALENT for v, _ in R[p]):
            V[p] = oracle.EQUIVALENT
        else:
            V[p] = oracle.UNDECIDED
    out = {
        "_about": "oracle/ results for every pair of workloads.c3_rand() (defaults); written by "
                  "scripts/make_golden_c3.py (support groups x pattern ranges, min-reduced)",
        "generator": "c3_rand", "kwargs": {},
        "num_pis": int(m.aig.num_pis), "num_ands": int(m.aig.num_ands),
        "lit_a": [int(x) for x in m.lit_a], "lit_b": [int(x) for x in m.lit_b],
        "verdict": V, "k": K, "cex": X,
        "oracle_node_evals": evals, "oracle_cpu_seconds": round(cpu_s, 1),
        "oracle_wall_seconds": round(time.time() - t0, 1), "oracle_processes": procs, "tasks": len(tasks),
    }
    with open(os.path.join(ROOT, "tests", "golden", "c3_rand.json"), "w") as fh:
        json.dump(out, fh)


if __name__ == "__main__":
    main()
