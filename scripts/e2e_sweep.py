"""End-to-end time of the public blocking call (cec_sim_exhaustive, host arrays in, verdicts out) under
different pipelining schedules (CEC_PIPE_FIRST = first chunk's share of the cost, CEC_PIPE_GROWTH =
chunk growth factor; csrc/cec_host.cpp). Median of `reps` calls per setting after one warm-up call.

  python scripts/e2e_sweep.py [c5] [reps]
"""
import json
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_dac_liuy25_b200 import capi  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "c5"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 7
m, _, _ = bench.make_workload(name)
merge = capi.CEC_MERGE_COST if name == "c3" else capi.CEC_MERGE_PAPER
stream = torch.cuda.Stream()
ctx = capi.Context.from_aig(m.aig, stream=stream.cuda_stream, merge=merge)
la, lb = np.ascontiguousarray(m.lit_a), np.ascontiguousarray(m.lit_b)
settings = [(None, None), ("0.02", "2"), ("0.02", "1.6"), ("0.01", "1.6"), ("0.03", "1.8"), ("0.04", "1.5"),
            ("0.015", "1.4")]
ref = None
for first, growth in settings:
    for k, v in (("CEC_PIPE_FIRST", first), ("CEC_PIPE_GROWTH", growth)):
        if v is None:
            os.environ.pop(k, None)
        else:
            os.environ[k] = v
    ctx.sim_exhaustive(la, lb)  # warm-up (JIT bundles of new chunkings compile here)
    ts = []
    for _ in range(reps):
        torch.cuda.synchronize()
        t = time.perf_counter()
        v, c, k = ctx.sim_exhaustive(la, lb)
        ts.append(1e3 * (time.perf_counter() - t))
        if ref is None:
            ref = (v, c)
        assert np.array_equal(v, ref[0]) and np.array_equal(c, ref[1])
    st = ctx.stats()
    print(json.dumps({"config": name, "first": first or "0.04 (default)", "growth": growth or "2 (default)",
                      "e2e_ms_median": statistics.median(ts), "e2e_ms_min": min(ts),
                      "kernel_ms": st["kernel_ms"], "host_prep_ms": st["host_prep_ms"],
                      "launches": st["num_launches"]}), flush=True)
