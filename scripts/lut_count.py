"""LUT (LOP3) count of the JIT mapping per AND node, host only (no GPU): plans the exhaustive sweep
in a host-only context (JIT programs are compiled, not loaded) and reports stats.lop3_words / W*32.
Usage: python scripts/lut_count.py [c5|c2|c3]   (CEC_JIT_FUSE selects the mapping mode)"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
from paper_conf_dac_liuy25_b200 import capi  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "c5"
m, _, _ = bench.make_workload(name)
merge = capi.CEC_MERGE_COST if name == "c3" else capi.CEC_MERGE_PAPER
ctx = capi.Context.from_aig(m.aig, device=-1, merge=merge, engine=int(os.environ.get("CEC_ENGINE", capi.CEC_ENGINE_JIT)))
t = time.perf_counter()
plan = capi.cec_plan_exhaustive(ctx.handle, m.lit_a, m.lit_b)
dt = time.perf_counter() - t
info = capi.cec_plan_info(plan)
st = ctx.stats()
print(st)
W = info["node_patterns"]
print(f"{name}: W={W:.4g} lop3_words={st['lop3_words']} lop3/and={st['lop3_words'] * 32 / W:.4f} "
      f"imad/and={st['imad_words'] * 32 / W:.4f} plan {dt:.1f}s")
capi.cec_plan_free(plan)
