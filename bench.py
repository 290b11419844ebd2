#!/usr/bin/env python
"""bench.py — AIG node-pattern evals/s of the exhaustive-simulation hot path on B200.

One "step" = one full cec_plan_run of the workload: every window's whole 2^k pattern space
simulated and every candidate pair compared, plus the cross-GPU min of
the first-mismatch indices when N > 1 (default: fused over NVLink peer memory, include/cec.h
cec_peer_export/import; --reduce nccl: one ncclAllReduce; the line's config.cross_gpu_reduce says
which ran). Default workload = C5 (BASELINE.json configs[4], the config the metric is
quoted on at 1/2/4/8 GPUs): 256 disjoint copies, ~2.1M ANDs, 6320 PO pairs, k = 24 per copy.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config c5|c3|c2|c2bug|c1] [--impl ours|reference]
                  [--reduce peer|nccl]

value      = W (node-patterns of one step, all ranks) / device time per step (CUDA events on the
             launch stream, max over ranks), schedules resident in HBM, L2 flushed between steps
e2e        = same metric through the public blocking C call cec_sim_exhaustive with host arrays
             (planning + H2D of schedules + kernels + all-reduce + D2H of results per step)
roofline   = ALU (LOP3) bound: the mapped window's lop3.b32 cells per u32 word (32 patterns) are the
             work of the binding pipe; peak = 148 SMs x 64 LOP3/clk/SM x SM clock.
             IMAD cells (AND nodes with a word-uniform operand, FMA pipe) are reported beside it.
cpu_baseline / --impl reference = the oracle (oracle/, plain single-threaded C) timed on a bounded
             sample of the same workload on this host's cores (one oracle process per core, each on
             its own pattern range: the sharded oracle of SURVEY.md §8(c)).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "AIG node-pattern evals/s"
WORKLOAD_SEEDS = {"c5": 5, "c3": 3, "c2bug": 1, "c2": None, "c1": None}  # generator seeds (workloads/circuits.py)
UNIT = "node-patterns/s"
LOP3_PER_CLK_PER_SM = 64  # alu pipe: rt = 2 cycles per warp-instr per SMSP, 4 SMSPs (B300_MICROARCH.md)


def make_workload(name: str):
    from workloads import c1_add8, c2_mul12, c2_mul12_bug, c3_rand, c5_big

    if name == "c5":
        m = c5_big()
        desc = ("c5_big2m: 256 disjoint copies (176 random-block sin_10xd-shaped miters of 3 types + 80 "
                "mul12 array-vs-Wallace miters), 8 seeded single-gate bug copies, 24 PIs per copy")
        return m, desc, 0  # copy index 0 for the oracle sample
    if name == "c2":
        return c2_mul12(), "c2_mul12: 12x12 array vs Wallace multiplier miter", None
    if name == "c2bug":
        return c2_mul12_bug(seed=1), "c2_mul12_bug1: C2 with one flipped complement in B's tree", None
    if name == "c3":
        return c3_rand(), ("c3_rand100k: 200 random blocks (~100k ANDs) vs rewritten copy over 1024 PIs; "
                           "1600 PO pairs + 5000 internal (A node, B image) pairs + 64 near-miss pairs"), None
    if name == "c1":
        return c1_add8(), "c1_add8: 8-bit ripple-carry vs Kogge-Stone adder miter", None
    raise SystemExit(f"unknown config {name}")


L2_NOTE = ("ours: L2 flushed between timed steps (256 MiB write, outside the events); "
           "reference arm: the CPU oracle, no GPU")


def workload_config(name, m, desc):
    """The `config` object of BOTH arms' JSON lines: it names the workload only (generator-derived
    facts, identical for --impl ours and --impl reference); run-specific facts (plan, engine, reduce
    mode) go to the line's `plan` object."""
    return {"workload": name, "description": desc, "pis": int(m.aig.num_pis), "ands": int(m.aig.num_ands),
            "pairs": int(m.num_pairs), "l2": L2_NOTE}


def sample_pairs(m, copy_idx):
    """Pairs of one copy (C5) or all pairs."""
    import numpy as np

    if copy_idx is None or "pairs_per_copy" not in m.meta:
        return m.lit_a, m.lit_b, "all pairs"
    off = int(np.sum(m.meta["pairs_per_copy"][:copy_idx]))
    n = m.meta["pairs_per_copy"][copy_idx]
    return m.lit_a[off:off + n], m.lit_b[off:off + n], f"the {n} PO pairs of copy {copy_idx}"


_SHARD = {}  # the oracle and pairs a forked shard process inherits


def _oracle_shard(rng):
    lo, hi = rng
    _, _, _, evals = _SHARD["orc"].check_pairs(_SHARD["la"], _SHARD["lb"], k_max=32, lo=lo, hi=hi)
    return evals


def host_cores():
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


def oracle_sample(m, copy_idx, log2_patterns, procs=1, reps=1):
    """Time the oracle (as it stands: single-threaded C) on one copy's pair group. procs > 1: the
    sharded oracle of SURVEY.md §8(c) — procs forked processes, one per host core, each enumerating
    its own 2^log2_patterns-pattern range of the window (min over ranges = the full scan); the
    timed region is the parallel map only (workers are forked and warmed before it)."""
    import multiprocessing

    import oracle

    la, lb, what = sample_pairs(m, copy_idx)
    orc = oracle.Oracle.from_aig(m.aig)
    n = 1 << log2_patterns
    if procs <= 1:
        evals, dt = 0, 0.0
        for _ in range(reps):
            t = time.perf_counter()
            _, _, _, e = orc.check_pairs(la, lb, k_max=32, lo=0, hi=n)
            dt += time.perf_counter() - t
            evals += e
        return evals, dt, f"{what}, patterns [0, 2^{log2_patterns}) of its 2^24-pattern window, single thread"
    _SHARD.update(orc=orc, la=la, lb=lb)
    try:  # forked after CUDA init: the workers only run the C oracle; bounded wait, else one thread
        with multiprocessing.get_context("fork").Pool(procs) as pool:
            pool.map_async(_oracle_shard, [(0, 1)] * procs).get(timeout=120)  # fork + warm, untimed
            evals, dt = 0, 0.0
            for _ in range(reps):
                t = time.perf_counter()
                evals += sum(pool.map_async(_oracle_shard, [(r * n, (r + 1) * n) for r in range(procs)],
                                            chunksize=1).get(timeout=600))
                dt += time.perf_counter() - t
    except Exception as e:  # pragma: no cover - safety net
        print(f"bench: sharded oracle failed ({e!r}); single-thread sample instead", file=sys.stderr)
        return oracle_sample(m, copy_idx, log2_patterns, 1, reps)
    return evals, dt, (f"{what}, patterns [0, {procs}*2^{log2_patterns}) of its 2^24-pattern window in {procs} "
                       f"ranges, one single-threaded oracle process per host core (SURVEY.md §8(c) sharded oracle)")


class ClockSampler:
    """SM clock + throttle reasons sampled DURING the timed region: an NVML polling thread (every
    5 ms, plus one sample on entry and one on exit so even a sub-millisecond region has readings)."""
    REASONS = {0x8: "hw_slowdown", 0x40: "hw_thermal_slowdown", 0x20: "sw_thermal_slowdown",
               0x4: "sw_power_cap", 0x80: "hw_power_brake_slowdown"}

    def __init__(self, gpu: int):
        self.gpu = gpu
        self.rows = []
        self.stop = None
        self.thread = None
        self.h = None
        self.nvml = None

    def _handle(self):
        import pynvml as nv
        nv.nvmlInit()
        self.nvml = nv
        try:  # the torch device's own PCI bus id (CUDA_VISIBLE_DEVICES may renumber)
            import torch
            p = torch.cuda.get_device_properties(self.gpu)
            bus = f"{p.pci_domain_id:08x}:{p.pci_bus_id:02x}:{p.pci_device_id:02x}.0"
            return nv.nvmlDeviceGetHandleByPciBusId(bus)
        except Exception:
            return nv.nvmlDeviceGetHandleByIndex(self.gpu)

    def _sample(self):
        nv = self.nvml
        sm = nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM)
        try:
            r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
        except Exception:
            r = nv.nvmlDeviceGetCurrentClocksThrottleReasons(self.h)
        try:
            pw = nv.nvmlDeviceGetPowerUsage(self.h) / 1e3
        except Exception:
            pw = None
        self.rows.append((sm, r, pw))

    def __enter__(self):
        try:
            self.h = self._handle()
            self.max_mhz = self.nvml.nvmlDeviceGetMaxClockInfo(self.h, self.nvml.NVML_CLOCK_SM)
            self._sample()
        except Exception:
            self.h = None
            return self
        self.stop = threading.Event()

        def loop():
            while not self.stop.wait(0.005):
                self._sample()

        self.thread = threading.Thread(target=loop, daemon=True)
        self.thread.start()
        return self

    def __exit__(self, *a):
        if self.thread:
            self._sample()
            self.stop.set()
            self.thread.join()

    def summary(self):
        if self.h is None or not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvml unavailable"]}
        sm = [r[0] for r in self.rows]
        reasons = sorted({name for _, bits, _ in self.rows for b, name in self.REASONS.items() if bits & b})
        pw = [r[2] for r in self.rows if r[2] is not None]
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": float(self.max_mhz), "reasons": reasons,
                "samples": len(self.rows), "source": "nvml 5 ms", "power_w_max": max(pw) if pw else None}


def run_reference(args):
    """--impl reference: the oracle as it stands, on rank 0's host cores, bounded sample per step."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle

    oracle.build()
    m, desc, copy_idx = make_workload(args.config)
    log2p = args.ref_log2_patterns
    procs = host_cores() if args.cpu_procs <= 0 else args.cpu_procs
    oracle_sample(m, copy_idx, log2p - 2, procs, reps=args.warmup)  # warm-up steps (smaller)
    evals, secs, what = oracle_sample(m, copy_idx, log2p, procs, reps=args.steps)
    v = evals / secs
    line = {
        "impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * secs / args.steps,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u8",
        "data": "synthetic",
        "config": workload_config(args.config, m, desc),
        "cpu_baseline": {"value": v, "unit": UNIT, "cores": procs, "kind": "oracle", "sample": what},
        "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="c5")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--engine", type=int, default=0, help="0 auto, 1 interpreter, 2 JIT, 3 paper Alg. 1 (simt in HBM)")
    ap.add_argument("--e2e-steps", type=int, default=5)
    ap.add_argument("--merge", type=int, default=-1, help="0 off, 1 paper (default), 2 cost-aware (default for c3)")
    ap.add_argument("--cpu-log2-patterns", type=int, default=19)
    ap.add_argument("--ref-log2-patterns", type=int, default=17)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-procs", type=int, default=0, help="oracle processes for cpu_baseline / reference (0 = host cores)")
    ap.add_argument("--reduce", default="peer", choices=["peer", "nccl"],
                    help="N > 1: a10 over NVLink peer memory fused into the compare path (default) or ncclAllReduce")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        return run_reference(args)

    import numpy as np
    import torch
    import torch.distributed as dist

    from paper_conf_dac_liuy25_b200 import capi

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # BENCH_SAME_GPU=1 (testing only): every rank on device 0, gloo process group, peer reduction only
    # (NCCL refuses two ranks on one GPU) with HOST barriers (cec_peer_host_barrier: kernels that wait
    # on one another must not share one GPU). Times are meaningless there (ranks time-slice one GPU).
    same_gpu = os.environ.get("BENCH_SAME_GPU") == "1"
    if same_gpu:
        local = 0
    torch.cuda.set_device(local)
    if world > 1:
        if same_gpu:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    red_dev = "cpu" if same_gpu else "cuda"

    def allreduce(x, op):
        t = torch.tensor([x], device=red_dev, dtype=torch.float64)
        dist.all_reduce(t, op=op)
        return float(t.item())

    stream = torch.cuda.Stream()  # the library launches on this stream; events are recorded on it
    torch.cuda.set_stream(stream)

    m, desc, copy_idx = make_workload(args.config)
    merge = args.merge if args.merge >= 0 else (capi.CEC_MERGE_COST if args.config == "c3" else capi.CEC_MERGE_PAPER)

    def new_uid():
        if world == 1 or same_gpu:
            return None
        obj = [capi.cec_nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        return obj[0]

    def all_gather(blob):
        out = [None] * world
        dist.all_gather_object(out, blob)
        return out

    def open_ctx(peer):
        """Context + plan + one checked run; peer=True: a10 over peer memory (include/cec.h
        cec_peer_export/import, IPC blobs all-gathered here), else ncclAllReduce. Every collective
        step is taken by every rank even after a local failure, so no rank waits for a failed one."""
        c = capi.Context.from_aig(m.aig, device=local, rank=rank, world=world, stream=stream.cuda_stream,
                                  engine=args.engine, merge=merge, nccl_unique_id=new_uid())
        err, pl = None, None
        if peer:
            blob = None
            try:
                blob = capi.cec_peer_export(c.handle)
            except capi.CecError as e:
                err = str(e)
            blobs = all_gather(blob)
            if all(b is not None for b in blobs):
                try:
                    capi.cec_peer_import(c.handle, blobs)
                    if same_gpu:  # ranks on one device never spin on each other (include/cec.h)
                        c._host_barrier_cb = capi.cec_peer_host_barrier(c.handle, dist.barrier)
                except capi.CecError as e:
                    err = str(e)
            else:
                err = err or "peer export failed on a peer rank"
        try:
            pl = capi.cec_plan_exhaustive(c.handle, m.lit_a, m.lit_b)  # JIT compiles: ranks skew here
        except capi.CecError as e:
            err = err or str(e)
        if world > 1 and allreduce(0.0 if err else 1.0, dist.ReduceOp.MIN) != 1.0:
            return c, pl, err or "a peer rank failed"
        try:
            capi.cec_plan_run(c.handle, pl)
            capi.cec_plan_results(c.handle, pl, m.num_pairs)  # syncs; raises on a barrier timeout
        except capi.CecError as e:
            err = str(e)
        return c, pl, err

    t_load = time.perf_counter()
    peer = world > 1 and (args.reduce == "peer" or same_gpu)
    ctx, plan, err = open_ctx(peer)
    load_ms = 1e3 * (time.perf_counter() - t_load)
    reduce_mode = "none (1 GPU)"
    if world > 1:
        ok = allreduce(0.0 if err else 1.0, dist.ReduceOp.MIN)  # every rank takes the same path
        if peer and ok == 1.0:
            reduce_mode = ("peer memory (one-GPU emulation: fused atomicMin into rank 0's home arrays + HOST barriers)"
                           if same_gpu else
                           "peer memory (NVLink, fused atomicMin into rank 0's home arrays + device barriers)")
        elif peer and not same_gpu:  # fall back to the collective on every rank
            ctx.close()
            ctx, plan, err2 = open_ctx(False)
            if err2:
                raise SystemExit(f"rank {rank}: {err2}")
            reduce_mode = "nccl all-reduce (min); peer mode failed" + (f": {err}" if err else " on a peer rank")
        elif ok != 1.0:
            raise SystemExit(f"rank {rank}: {err or 'a peer rank failed'}")
        else:
            reduce_mode = "nccl all-reduce (min)"
    elif err:
        raise SystemExit(err)
    info = capi.cec_plan_info(plan)
    st0 = ctx.stats()
    engine_name = ("simt (paper Alg. 1)" if args.engine == capi.CEC_ENGINE_SIMT else
                   "jit" if st0["jit_windows"] == info["num_windows"] else
                   "interp" if st0["jit_windows"] == 0 else f"jit({st0['jit_windows']} windows)+interp")

    for _ in range(args.warmup):
        capi.cec_plan_run(ctx.handle, plan)
    torch.cuda.synchronize()
    v, cex, k = capi.cec_plan_results(ctx.handle, plan, m.num_pairs)
    verdicts = {"EQ": int((v == capi.CEC_EQUIVALENT).sum()), "NEQ": int((v == capi.CEC_NOT_EQUIVALENT).sum()),
                "UND": int((v == capi.CEC_UNDECIDED).sum())}
    stats = ctx.stats()
    W_rank, W_all = stats["node_patterns"], stats["node_patterns_all"]
    launches_per_step = stats["num_launches"]

    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    starts = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    ends = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        t0 = time.perf_counter()
        for i in range(args.steps):
            flush.zero_()  # L2 flush between timed steps (outside the events)
            starts[i].record(stream)
            capi.cec_plan_run(ctx.handle, plan)
            ends[i].record(stream)
        torch.cuda.synchronize()
        wall = time.perf_counter() - t0
        # the window kernels' own device time: the same K steps again with CUDA events around the
        # window kernels (include/cec.h cec_plan_sweep_timing / _ms; off in the steps above, where
        # the two event nodes would add ~7 us to a small config's captured run)
        sweep_ms = []
        if args.engine != capi.CEC_ENGINE_SIMT:
            capi.cec_plan_sweep_timing(plan, True)
            capi.cec_plan_run(ctx.handle, plan)  # recapture with the event nodes (untimed)
            for i in range(args.steps):
                flush.zero_()
                capi.cec_plan_run(ctx.handle, plan)
                torch.cuda.synchronize()
                sweep_ms.append(capi.cec_plan_sweep_ms(plan))
            capi.cec_plan_sweep_timing(plan, False)
    if world > 1:
        dist.barrier()
    step_ms = [s.elapsed_time(e) for s, e in zip(starts, ends)]
    ms = sum(step_ms) / len(step_ms)
    if world > 1:
        ms = allreduce(ms, dist.ReduceOp.MAX)
    value = W_all / (ms / 1e3)

    # e2e: the public blocking call with host arrays (plan + H2D + kernels + reduce + D2H)
    e2e_ms = []
    la_h, lb_h = np.ascontiguousarray(m.lit_a), np.ascontiguousarray(m.lit_b)
    # one untimed call first: the pipelined call plans windows in chunks whose JIT bundles are
    # compiled (and cached) on first use; compile time is reported separately, never timed
    t = time.perf_counter()
    ctx.sim_exhaustive(la_h, lb_h)
    e2e_warm_ms = 1e3 * (time.perf_counter() - t)
    e2e_jit_ms = ctx.stats()["jit_ms"]
    for _ in range(max(1, args.e2e_steps)):
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        t = time.perf_counter()
        ve, ce, ke = ctx.sim_exhaustive(la_h, lb_h)
        e2e_ms.append(1e3 * (time.perf_counter() - t))
        assert np.array_equal(ve, v) and np.array_equal(ce, cex)
    st_e2e = ctx.stats()
    e2e = statistics.median(e2e_ms)
    if world > 1:
        e2e = allreduce(e2e, dist.ReduceOp.MAX)

    clocks = clk.summary()
    sm_clock = clocks.get("sm_mhz") or clocks.get("sm_max_mhz") or 1965.0  # median SM clock seen under load
    props = torch.cuda.get_device_properties(local)
    peak = props.multi_processor_count * LOP3_PER_CLK_PER_SM * sm_clock * 1e6 / 1e12  # TLOP3/s
    # algorithmic LOP3s of the path: one 3-input LUT per mapped node group per u32 word (JIT), one
    # per AND (interpreter) — the AND-node count itself is the metric W — over the window kernels'
    # own device time per launch (CUDA events around them on the launch stream, mean over the
    # second pass of K steps; the step adds the reset kernel and the graph launch); step_frac is
    # the same rate over the timed step
    kern_ms = statistics.mean(sweep_ms) if sweep_ms else ms
    if world > 1:
        kern_ms = allreduce(kern_ms, dist.ReduceOp.MAX)
    achieved = stats["lop3_words"] / (kern_ms / 1e3) / 1e12
    simt = args.engine == capi.CEC_ENGINE_SIMT
    traffic = None
    prof = os.path.join(ROOT, "profiles", "ncu_summary.json")
    if os.path.exists(prof):
        try:
            traffic = json.load(open(prof)).get(args.config, {}).get("dram_bytes_per_launch")
        except Exception:
            traffic = None

    hbm_peak = 6453.7
    mp = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(mp):
        try:
            hbm_peak = float(json.load(open(mp)).get("hbm_gbs", hbm_peak))
        except Exception:
            pass
    simt_gbs = 12.0 * (W_rank / 32.0) / (ms / 1e3) / 1e9
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        import oracle

        oracle.build()
        procs = host_cores() if args.cpu_procs <= 0 else args.cpu_procs
        evals, dt, what = oracle_sample(m, copy_idx, args.cpu_log2_patterns, procs)
        cpu = {"value": evals / dt, "unit": UNIT, "cores": procs, "kind": "oracle", "sample": what,
               "seconds": round(dt, 2)}

    # parity against stored oracle results of the same generated miter (tests/golden, written by
    # scripts/make_golden*.py, which call only oracle/): every pair's verdict, k and canonical CEX
    parity = None
    gold_name = {"c5": "c5_big", "c3": "c3_rand", "c2": "c2_mul12", "c2bug": "c2_mul12_bug1",
                 "c1": "c1_add8"}.get(args.config)
    gpath = os.path.join(ROOT, "tests", "golden", f"{gold_name}.json") if gold_name else None
    if rank == 0 and gpath and os.path.exists(gpath):
        g = json.load(open(gpath))
        if g["lit_a"] == [int(x) for x in m.lit_a] and g["lit_b"] == [int(x) for x in m.lit_b]:
            gv, gk = np.array(g["verdict"]), np.array(g["k"])
            gc = np.array([int(x) for x in g["cex"]], dtype=np.uint64)
            neq = gv == capi.CEC_NOT_EQUIVALENT
            diffs = int((gv != v).sum() + (gk != k).sum() + (neq & (gc != cex)).sum())
            parity = {"vs": f"tests/golden/{gold_name}.json (oracle/, every pair)", "pairs": int(gv.size),
                      "diffs": diffs, "ok": diffs == 0}

    # SURVEY.md §8(d) "Runs and reporting": the per-run record under the survey's own field names
    h2d_ms = None
    if st_e2e["h2d_bytes"]:  # one pinned host -> device copy of the call's H2D bytes, CUDA events
        hb = torch.empty(int(st_e2e["h2d_bytes"]), dtype=torch.uint8, pin_memory=True)
        db = torch.empty_like(hb, device="cuda")
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        db.copy_(hb, non_blocking=True)
        e0.record(stream)
        db.copy_(hb, non_blocking=True)
        e1.record(stream)
        torch.cuda.synchronize()
        h2d_ms = e0.elapsed_time(e1)
    ncu = {}
    if os.path.exists(prof):
        try:
            ncu = json.load(open(prof)).get(args.config, {})
        except Exception:
            ncu = {}
    record = {
        "config": args.config, "seed": WORKLOAD_SEEDS.get(args.config), "gpus": world, "W": W_all,
        "t_kernel_ms": statistics.median(step_ms), "node_patterns_per_s": value, "t_e2e_ms": e2e,
        "t_hostprep_ms": st_e2e["host_prep_ms"], "t_h2d_ms": h2d_ms,
        "t_allreduce_us": 1e3 * max(0.0, ms - kern_ms) if world > 1 else 0.0,
        "dram_GBps": (ncu["dram_bytes_per_launch"] / ncu["profiled_launch_ns"]
                      if ncu.get("dram_bytes_per_launch") and ncu.get("profiled_launch_ns") else None),
        "alu_pipe_pct": ncu.get("alu_pipe_pct"),
        "lop3_count_per_W32": stats["lop3_words"] / max(1.0, W_rank / 32.0),
        "sm_clock_MHz": sm_clock,
        "oracle_wall_s": cpu["seconds"] if cpu else None, "oracle_cores": cpu["cores"] if cpu else None,
        "oracle_cpu_s": cpu["seconds"] * cpu["cores"] if cpu else None,
        "parity": parity,
        "notes": ("t_kernel_ms: median step; t_h2d_ms: one pinned copy of the call's H2D bytes; "
                  "t_allreduce_us: step minus window-kernel time (reset + reduction + launch), N > 1; "
                  "dram_GBps / alu_pipe_pct: ncu --set full of one window kernel of this config "
                  f"(profiles/ncu_summary.json, {ncu.get('source', 'none')})"),
    }

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": workload_config(args.config, m, desc),
            "plan": {"windows": info["num_windows"], "max_k": info["max_k"],
                       "max_slots": info["max_slots"], "node_patterns_per_step": W_all,
                       "parallelism": f"pattern-space shards x{world}", "cross_gpu_reduce": reduce_mode,
                       "merge": ["off", "paper", "cost-aware"][merge], "engine": engine_name, "jit_kernels": st0["jit_kernels"], "jit_compile_ms": st0["jit_ms"],
                       "verdicts": verdicts},
            "clocks": clocks,
            "parity": parity,
            "record": record,
            "gpu_launches": int(launches_per_step * args.steps),
            "e2e": {"value": W_all / (e2e / 1e3), "unit": UNIT, "ms_per_miter": e2e,
                    "h2d_bytes_per_step": int(st_e2e["h2d_bytes"]), "d2h_bytes_per_step": int(st_e2e["d2h_bytes"]),
                    "host_prep_ms": st_e2e["host_prep_ms"], "device_ms": st_e2e["kernel_ms"],
                    "context_open_ms": load_ms,  # AIG load + first plan (JIT compiles) + one checked run
                    "warmup_call_ms": round(e2e_warm_ms, 2), "warmup_jit_compile_ms": round(e2e_jit_ms, 2)},
            "roofline": ({"bound": "hbm", "achieved": simt_gbs, "peak": hbm_peak, "unit": "GB/s",
                          "frac": simt_gbs / hbm_peak, "traffic": None,
                          "peak_basis": "MEASURED_PEAKS.json hbm_gbs (copy bandwidth)",
                          "algorithmic_bytes": "12 B per node per u32 word (2 fanin reads + 1 write of the simulation table)"}
                         if simt else
                         {"bound": "alu", "achieved": achieved, "peak": peak, "unit": "TLOP3/s",
                         "frac": achieved / peak, "traffic": traffic,
                         "kernel_ms": kern_ms, "kernel_timing": "CUDA events around the window kernels "
                         "(cec_plan_sweep_ms), mean over a second pass of the K steps",
                         "step_frac": stats["lop3_words"] / (ms / 1e3) / 1e12 / peak,
                         "peak_basis": f"{props.multi_processor_count} SMs x {LOP3_PER_CLK_PER_SM} LOP3/clk x {sm_clock:.0f} MHz (guide unit counts, SM clock; microbenchmark scripts/peaks.cu measured 64.00 LOP3/clk/SM = 18.53 TLOP3/s at 1957 MHz, profiles/round1_peaks.json)",
                         "lop3_per_word_per_and": stats["lop3_words"] / max(1.0, W_rank / 32.0),
                         "imad_per_word_per_and": stats.get("imad_words", 0) / max(1.0, W_rank / 32.0),
                         "fma_pipe_timad_s": stats.get("imad_words", 0) / (kern_ms / 1e3) / 1e12,
                         "cells": "3-input LUTs = lop3.b32 on the ALU pipe (the bound); AND nodes with a "
                                  "word-uniform operand = mad.lo.u32 on the FMA pipe (DESIGN.md §4.1)",
                         "and_evals_tops": (W_rank / 32.0) / (kern_ms / 1e3) / 1e12,
                         # the SURVEY §8(d) unit (one 2-input op per AND per u32 word) against the same
                         # peak: > 1 because a mapped LOP3/IMAD cell evaluates ~1.9 ANDs
                         "and_evals_per_lop3_peak": (W_rank / 32.0) / (kern_ms / 1e3) / 1e12 / peak}),
            "step_ms": step_ms, "wall_s": wall,
        }
        if cpu:
            line["cpu_baseline"] = cpu
        print(json.dumps(line), flush=True)
    capi.cec_plan_free(plan)
    ctx.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
