"""N > 1 path on CPU (gloo, world_size 2): pattern-space sharding of SURVEY.md §8(e).

Each rank plans the same miter with rank/world set (host-only context: no GPU here), so the
partition of every window's slices and the per-rank work W are exercised; the min-reduction of
first-mismatch indices is exercised with the oracle run on each rank's pattern range, reduced by
torch.distributed (gloo) exactly as ncclAllReduce(min) reduces the GPU indices."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

NO = (1 << 64) - 1


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        import oracle
        from paper_conf_dac_liuy25_b200 import capi
        from workloads import circuits

        m = circuits.c2_mul12_bug(seed=1, n=7)
        # (1) host planning per rank: shard W adds up to the whole
        ctx = capi.Context.from_aig(m.aig, device=-1, rank=rank, world=world)
        plan = capi.cec_plan_exhaustive(ctx.handle, m.lit_a, m.lit_b)
        st = ctx.stats()
        w = torch.tensor([st["node_patterns"]], dtype=torch.float64)
        dist.all_reduce(w, op=dist.ReduceOp.SUM)
        ok_w = int(w.item()) == st["node_patterns_all"]
        capi.cec_plan_free(plan)
        # (2) min-reduction of first-mismatch indices over pattern-range shards (oracle per rank)
        orc = oracle.Oracle.from_aig(m.aig)
        v_full, c_full, k_full, _ = orc.check_pairs(m.lit_a, m.lit_b)
        firsts = []
        for p in range(m.num_pairs):
            total = 1 << int(k_full[p])
            b, e = capi.cec_shard_range(total, rank, world)
            vs, cs, _, _ = orc.check_pairs(m.lit_a[p:p + 1], m.lit_b[p:p + 1], lo=b, hi=e)
            firsts.append(int(cs[0]) if vs[0] == oracle.NOT_EQUIVALENT else -1)
        # NO_CEX as int64 max for the MIN reduction
        t = torch.tensor([f if f >= 0 else (1 << 62) for f in firsts], dtype=torch.int64)
        dist.all_reduce(t, op=dist.ReduceOp.MIN)
        red = [int(x) for x in t]
        want = [int(c) if v == oracle.NOT_EQUIVALENT else (1 << 62) for v, c in zip(v_full, c_full)]
        q.put((rank, ok_w, red == want))
        dist.destroy_process_group()
    except Exception as e:  # surface failures to the parent
        q.put((rank, False, repr(e)))


@pytest.mark.parametrize("world", [2])
def test_gloo_sharding_and_min_reduce(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    for rank, ok_w, ok_red in res:
        assert ok_w is True, (rank, ok_w, ok_red)
        assert ok_red is True, (rank, ok_red)
