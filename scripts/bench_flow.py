"""Measurement of the §8(f) rows around the hot path on B200 (one JSON line per row and config):

  NEXT-2  cec_sim_classes : partial simulation (random words) + exact equivalence classes + pairs
  NEXT-3  cec_reduce      : miter reduction (merge + strash rebuild)
  a12     cec_check_local_cuts on the local checks the C4 flow issues in its first L phase
          (config "c4"): node-patterns/s and the LOP3-pipe fraction of the interpreter kernel

Each row reports the median wall time of the blocking C-ABI call (host schedule, H2D of the merge
list / D2H of the results included) and the median device time of its kernels (CUDA events on the
launch stream, stats.kernel_ms) over --reps calls after one warm-up, on the configuration's full
AIG; the roofline fraction uses the device time. `roofline` is the HBM bound of the algorithmic bytes (classes: every node row of W words is
written once and its two fanin rows read once, then read again for the signature: 16 B per
node-word; reduce: per AND 8 B fanins + 4 B merge entry + 2 x 4 B fanin images + 4 B image + a
16 B table probe ~= 40 B) against MEASURED_PEAKS' HBM copy bandwidth. The oracle
(oracle/classes.py, oracle/reduce.py; single thread) is timed on the same input beside it.

Usage: python scripts/bench_flow.py [--configs c3,c5] [--reps 5] [--words 64]
"""
import argparse
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

from paper_conf_dac_liuy25_b200 import capi  # noqa: E402


def hbm_peak():
    try:
        d = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
        for k in ("hbm_gbs", "hbm_copy_GBps", "hbm_GBps"):
            if k in d:
                return float(d[k]), "MEASURED_PEAKS.json:" + k
        for k, v in d.items():
            if "hbm" in k.lower() and isinstance(v, (int, float)):
                return float(v), "MEASURED_PEAKS.json:" + k
    except Exception:
        pass
    return 6453.7, "SURVEY.md §8(d) copy bandwidth"


def timed(fn, ctx, reps):
    """(median call wall time, median device time of the call's kernels from stats.kernel_ms)."""
    fn()
    ts, ks = [], []
    for _ in range(reps):
        t = time.perf_counter()
        fn()
        ts.append(time.perf_counter() - t)
        ks.append(ctx.stats()["kernel_ms"] / 1e3)
    return statistics.median(ts), statistics.median(ks)


def po_merges(m):
    subst = {}
    for a, b in zip(m.lit_a, m.lit_b):
        hi, lo = (int(a), int(b)) if (a >> 1) > (b >> 1) else (int(b), int(a))
        if (hi >> 1) > m.aig.num_pis and (hi >> 1) != (lo >> 1) and (hi >> 1) not in subst:
            subst[hi >> 1] = lo ^ (hi & 1)
    return subst


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="c3,c5")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--words", type=int, default=64)
    ap.add_argument("--no-oracle", action="store_true")
    a = ap.parse_args()
    import bench
    import oracle
    from oracle.classes import classes as oracle_classes
    from oracle.reduce import reduce_miter

    peak, peak_src = hbm_peak()
    for name in a.configs.split(","):
        if name == "c4":
            local_row(a)
            continue
        m, _, _ = bench.make_workload(name)
        N = m.aig.num_nodes
        ctx = capi.Context.from_aig(m.aig, device=0)
        # ---- NEXT-2: classes
        out = {}
        t, tk = timed(lambda: out.__setitem__("c", ctx.sim_classes(a.words, 1)), ctx, a.reps)
        npairs = int(out["c"][0].size)
        bytes_alg = 16.0 * N * a.words * 1.0
        rec = {"row": "NEXT-2 cec_sim_classes", "config": name, "nodes": N, "words": a.words,
               "pairs": npairs, "call_ms": round(1e3 * t, 3), "kernel_ms": round(1e3 * tk, 3),
               "launches": ctx.stats()["num_launches"],
               "roofline": {"bound": "hbm", "algorithmic_bytes": bytes_alg, "achieved_GBps": bytes_alg / tk / 1e9,
                            "peak_GBps": peak, "peak_source": peak_src, "frac": bytes_alg / tk / 1e9 / peak}}
        if not a.no_oracle:
            orc = oracle.Oracle.from_aig(m.aig)
            W_or = max(1, a.words // 16) if N > 1_000_000 else a.words
            t0 = time.perf_counter()
            ref = oracle_classes(orc, W_or, 1)
            rec["oracle"] = {"seconds": round(time.perf_counter() - t0, 2), "words": W_or, "cores": 1,
                             "kind": "oracle/classes.py", "pairs": len(ref)}
            if W_or == a.words:
                got = [(int(x), int(y), int(z)) for x, y, z in zip(*out["c"])]
                rec["parity"] = got == ref
        print(json.dumps(rec), flush=True)
        # ---- NEXT-3: reduction (the P-phase merges: every B-side PO into its A-side partner)
        subst = po_merges(m)
        mem = np.fromiter(subst.keys(), dtype=np.uint32, count=len(subst))
        rep = np.fromiter(subst.values(), dtype=np.uint32, count=len(subst))
        lits = np.concatenate([m.lit_a, m.lit_b])
        t, tk = timed(lambda: out.__setitem__("r", ctx.reduce(mem, rep, lits)), ctx, a.reps)
        A = m.aig.num_ands
        bytes_alg = 40.0 * A
        rec = {"row": "NEXT-3 cec_reduce", "config": name, "ands": A, "merges": len(subst),
               "new_ands": int(out["r"][0].shape[0]), "call_ms": round(1e3 * t, 3), "kernel_ms": round(1e3 * tk, 3),
               "host_schedule_ms": round(ctx.stats()["host_prep_ms"], 3), "launches": ctx.stats()["num_launches"],
               "roofline": {"bound": "hbm", "algorithmic_bytes": bytes_alg, "achieved_GBps": bytes_alg / tk / 1e9,
                            "peak_GBps": peak, "peak_source": peak_src, "frac": bytes_alg / tk / 1e9 / peak}}
        if not a.no_oracle:
            fan = [(int(x), int(y)) for x, y in m.aig.fanins]
            t0 = time.perf_counter()
            ofan, oimg, olits = reduce_miter(m.aig.num_pis, fan, subst, [int(x) for x in lits])
            rec["oracle"] = {"seconds": round(time.perf_counter() - t0, 2), "cores": 1, "kind": "oracle/reduce.py"}
            rec["parity"] = (np.array_equal(out["r"][0], np.array(ofan, dtype=np.uint32).reshape(-1, 2)) and
                             np.array_equal(out["r"][1], np.array(oimg, dtype=np.uint32)) and
                             np.array_equal(out["r"][2], np.array(olits, dtype=np.uint32)))
        print(json.dumps(rec), flush=True)
        ctx.close()


def local_row(a):
    """a12 on C4: the (pair, cut) checks of the flow's first G+L phase, replayed through the C-ABI."""
    import oracle
    from paper_conf_dac_liuy25_b200 import driver
    from workloads import c4_dp
    m = c4_dp(64)
    r = driver.check_miter(m.aig, m.lit_a, m.lit_b, driver.CecParams(k_l=16, C=16))
    v0 = [ch for ch in r.checks if ch["version"] == 0]
    aig = r.versions[0]
    la = np.array([ch["lit_a"] for ch in v0], dtype=np.uint32)
    lb = np.array([ch["lit_b"] for ch in v0], dtype=np.uint32)
    off, leaves = [0], []
    for ch in v0:
        leaves += ch["leaves"]
        off.append(len(leaves))
    ctx = capi.Context.from_aig(aig, device=0, k_max=16)
    out = {}
    t, tk = timed(lambda: out.__setitem__("v", ctx.check_local_cuts(la, lb, off, leaves)), ctx, a.reps)
    st = ctx.stats()
    W = st["node_patterns"]
    lop3 = st["lop3_words"]
    sm_mhz = 1965.0
    lop_peak = 148 * 64 * sm_mhz * 1e6
    rec = {"row": "a12 cec_check_local_cuts", "config": "c4 first L phase", "checks": int(la.size),
           "max_leaves": int(max(len(ch["leaves"]) for ch in v0)), "node_patterns": int(W),
           "call_ms": round(1e3 * t, 3), "kernel_ms": round(1e3 * tk, 3), "host_prep_ms": round(st["host_prep_ms"], 3),
           "node_patterns_per_s_kernel": W / tk, "node_patterns_per_s_call": W / t,
           "roofline": {"bound": "alu", "achieved_tlop3": lop3 / tk / 1e12, "peak_tlop3": lop_peak / 1e12,
                        "frac": lop3 / tk / lop_peak, "peak_basis": "148 SMs x 64 LOP3/clk x 1965 MHz"}}
    if not a.no_oracle:
        orc = oracle.Oracle.from_aig(aig)
        t0 = time.perf_counter()
        want = orc.check_local(la, lb, off, leaves)
        rec["oracle"] = {"seconds": round(time.perf_counter() - t0, 3), "cores": 1, "kind": "oracle.check_local",
                         "node_patterns_per_s": W / max(1e-9, time.perf_counter() - t0)}
        rec["parity"] = bool(np.array_equal(np.asarray(out["v"]), np.asarray(want)))
    print(json.dumps(rec), flush=True)
    ctx.close()


if __name__ == "__main__":
    main()
