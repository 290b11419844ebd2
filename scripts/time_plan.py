"""Host-side phase times of the public call (CEC_TIMING=1 makes libcec print one line per phase on
stderr). Usage: python scripts/time_plan.py [c5|c3|c2] [calls]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("CEC_TIMING", "1")

import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_dac_liuy25_b200 import capi  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "c5"
calls = int(sys.argv[2]) if len(sys.argv) > 2 else 4
m, _, _ = bench.make_workload(name)
merge = capi.CEC_MERGE_COST if name == "c3" else capi.CEC_MERGE_PAPER
stream = torch.cuda.Stream()
t = time.perf_counter()
ctx = capi.Context.from_aig(m.aig, stream=stream.cuda_stream, merge=merge)
print(f"load {1e3 * (time.perf_counter() - t):.2f} ms  cores {len(os.sched_getaffinity(0))}", file=sys.stderr)
la, lb = np.ascontiguousarray(m.lit_a), np.ascontiguousarray(m.lit_b)
for i in range(calls):
    torch.cuda.synchronize()
    t = time.perf_counter()
    ctx.sim_exhaustive(la, lb)
    st = ctx.stats()
    print(f"--- call {i}: {1e3 * (time.perf_counter() - t):.2f} ms (host_prep {st['host_prep_ms']:.2f}, "
          f"kernel {st['kernel_ms']:.2f})", file=sys.stderr, flush=True)
