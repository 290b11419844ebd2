import sys, time
sys.path.insert(0, '/root/repo')
import numpy as np
import torch
from paper_conf_dac_liuy25_b200 import capi
from workloads import c4_dp
m = c4_dp(64)
ts_open, ts_work, ts_close = [], [], []
for i in range(30):
    t = time.perf_counter(); ctx = capi.Context.from_aig(m.aig, k_max=16); t1 = time.perf_counter()
    ctx.sim_classes(8, i); ctx.sim_exhaustive(m.lit_a[:8], m.lit_b[:8]); t2 = time.perf_counter()
    ctx.close(); t3 = time.perf_counter()
    ts_open.append(t1 - t); ts_work.append(t2 - t1); ts_close.append(t3 - t2)
f = lambda v: "med %.2f ms max %.2f ms" % (1e3 * np.median(v), 1e3 * max(v))
print("open", f(ts_open)); print("work", f(ts_work)); print("close", f(ts_close))
