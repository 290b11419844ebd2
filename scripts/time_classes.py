import sys, time
sys.path.insert(0, '/root/repo')
import torch
from paper_conf_dac_liuy25_b200 import capi
from workloads import c5_big
m = c5_big()
ctx = capi.Context.from_aig(m.aig)
for i in range(8):
    torch.cuda.synchronize()
    t = time.perf_counter(); r = ctx.sim_classes(64, 1); dt = time.perf_counter() - t
    st = ctx.stats()
    print("call %.2f ms kernel %.2f ms pairs %d" % (dt * 1e3, st["kernel_ms"], len(r[0])), flush=True)
cap = len(r[0])
for i in range(4):
    t = time.perf_counter(); r = ctx.sim_classes(64, 1, cap=cap); dt = time.perf_counter() - t
    print("with cap: call %.2f ms" % (dt * 1e3), flush=True)
