"""Strong-scaling projection of bench.py's C5 step on ONE B200 (there is no multi-GPU box here).

For G in (1, 2, 4, 8) and every rank r < G: a context in shard-only mode (world = G, rank = r, no
NCCL id: DESIGN.md §6) plans C5 exactly as rank r of a G-GPU run would and its cec_plan_run is timed
with CUDA events (same L2 flush between steps as bench.py). The projected G-GPU step time is the
max over ranks (+ the all-reduce latency, not emulated: one 8 B x 6320-pair ncclAllReduce, ~10-30 us
over NVSwitch); projected speed-up S(G) = t(1) / max_r t_r(G).

  python scripts/scale_emulate.py [--config c5] [--steps 5] [--gpus 1,2,4,8]
Prints one JSON line per G.
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c5")
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--gpus", default="1,2,4,8")
    args = ap.parse_args()

    import torch

    import bench
    from paper_conf_dac_liuy25_b200 import capi

    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    m, _, _ = bench.make_workload(args.config)
    merge = capi.CEC_MERGE_COST if args.config == "c3" else capi.CEC_MERGE_PAPER
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    t1 = None
    for G in [int(x) for x in args.gpus.split(",")]:
        per_rank = []
        W_all = None
        for r in range(G):
            ctx = capi.Context.from_aig(m.aig, device=0, rank=r, world=G, stream=stream.cuda_stream, merge=merge)
            plan = capi.cec_plan_exhaustive(ctx.handle, m.lit_a, m.lit_b)
            for _ in range(args.warmup):
                capi.cec_plan_run(ctx.handle, plan)
            torch.cuda.synchronize()
            ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
            for s, e in ev:
                flush.zero_()
                s.record(stream)
                capi.cec_plan_run(ctx.handle, plan)
                e.record(stream)
            torch.cuda.synchronize()
            ms = sorted(s.elapsed_time(e) for s, e in ev)[len(ev) // 2]
            st = ctx.stats()
            W_all = st["node_patterns_all"]
            per_rank.append({"rank": r, "ms": round(ms, 3), "node_patterns": st["node_patterns"],
                             "launches": st["num_launches"]})
            capi.cec_plan_free(plan)
            ctx.close()
        tmax = max(p["ms"] for p in per_rank)
        if G == 1:
            t1 = tmax
        line = {"config": args.config, "gpus": G, "emulated": "each rank's shard timed alone on one B200",
                "max_rank_ms": tmax, "projected_value": W_all / (tmax / 1e3),
                "projected_speedup": (t1 / tmax) if t1 else None,
                "rank_balance": tmax / (sum(p["ms"] for p in per_rank) / G), "ranks": per_rank}
        print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
