"""Per-launch-group timing of one plan run (CEC_PROFILE_GROUPS=1: serial launches, CUDA events per
group, printed by libcec on stderr). Usage: python scripts/profile_groups.py [c3|c5|c2] [merge]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["CEC_PROFILE_GROUPS"] = "1"

import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_dac_liuy25_b200 import capi  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "c3"
merge = int(sys.argv[2]) if len(sys.argv) > 2 else (capi.CEC_MERGE_COST if name == "c3" else capi.CEC_MERGE_PAPER)
m, _, _ = bench.make_workload(name)
stream = torch.cuda.Stream()
ctx = capi.Context.from_aig(m.aig, stream=stream.cuda_stream, merge=merge)
plan = capi.cec_plan_exhaustive(ctx.handle, m.lit_a, m.lit_b)
for i in range(3):
    print(f"--- run {i}", file=sys.stderr, flush=True)
    capi.cec_plan_run(ctx.handle, plan)
    torch.cuda.synchronize()
capi.cec_plan_free(plan)
