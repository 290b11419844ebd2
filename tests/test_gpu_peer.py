"""GPU tests of the peer-memory cross-GPU reduction (include/cec.h cec_peer_export/import;
csrc/peer.cu; SURVEY.md §8(e) "B200-native option", §8(f) NEXT-4).

The box has one GPU, so `world` ranks are emulated as `world` PROCESSES on device 0, each with its
own CUDA context (time-sliced by the driver), exchanging CUDA IPC handles over a gloo process group —
the same cross-process mapping a one-process-per-GPU run uses. Kernels that wait on one another must
not run as separate launches on one GPU (B200_PROFILING.md: such ranks raised Xid 109), so the
emulated ranks replace the device barriers by host barriers (cec_peer_host_barrier: drain the stream,
then a gloo dist.barrier()); the rest of the peer path is the real one — IPC mappings, every rank's
window kernels doing system-scope atomicMin into rank 0's home arrays, cross-rank early-exit
bounds, the gather. Every rank must return exactly the single-GPU result — the same per-pair minimum
index the NCCL all-reduce produces (min over a partition of an ascending scan) — checked against the
oracle (bit-exact verdicts, k, canonical CEX). The device barrier kernel itself runs here only
alone (its timeout path), never against another rank's kernel."""
import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from oracle import Oracle  # noqa: E402
from paper_conf_dac_liuy25_b200 import capi  # noqa: E402
from workloads import c2_mul12_bug, c5_big, tiny_random  # noqa: E402

from test_gpu_parity import assert_same  # noqa: E402


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def _workload(name):
    if name == "c2bug10":
        return c2_mul12_bug(seed=1, n=10)
    if name == "c5small":
        return c5_big(copies=8, n_random=5, n_bugs=3, rand_pis=16, rand_ands=1500, mul_n=8)
    if name == "tiny":
        return tiny_random(9, 90, 24, 7011)
    if name == "tiny_local":
        return tiny_random(8, 60, 16, 505)
    raise KeyError(name)


def _local_cuts(m):
    """cut = each pair's own support (cut = S gives local EQ <=> global EQ)."""
    ref = capi.Context.from_aig(m.aig, device=-1)
    off, leaves = [0], []
    for a, b in zip(m.lit_a, m.lit_b):
        leaves += capi.cec_pair_support(ref.handle, int(a), int(b))
        off.append(len(leaves))
    return np.array(off, np.uint32), np.array(leaves, np.uint32)


def _lists(res):
    return [np.asarray(x).tolist() for x in res]


def _proc(rank, world, port, q, kind, name, engine):
    """One rank = one process with its own CUDA context on device 0 (as on a multi-GPU box, where it
    would be its own GPU): peer blocks mapped with cudaIpcOpenMemHandle, blobs over gloo."""
    import torch.distributed as dist

    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        m = _workload(name)
        ctx = capi.Context.from_aig(m.aig, device=0, rank=rank, world=world, engine=engine)

        def all_gather(blob):
            out = [None] * world
            dist.all_gather_object(out, blob)
            return out

        ctx.peer_connect(all_gather, host_barrier=dist.barrier)
        if kind == "sim":  # two blocking calls (the second reuses pools and JIT kernels)
            out = [_lists(ctx.sim_exhaustive(m.lit_a, m.lit_b)) for _ in range(2)]
            neq = [int(p) for p in np.nonzero(np.array(out[0][0]) == capi.CEC_NOT_EQUIVALENT)[0][:4]]
            out = (out, neq, [ctx.get_cex(p).tolist() for p in neq])
        elif kind == "plan":  # 4 runs of one plan: the 2nd on is a CUDA-graph replay
            plan = capi.cec_plan_exhaustive(ctx.handle, m.lit_a, m.lit_b)
            out = []
            for _ in range(4):
                capi.cec_plan_run(ctx.handle, plan)
                out.append(_lists(capi.cec_plan_results(ctx.handle, plan, m.num_pairs)))
            capi.cec_plan_free(plan)
        elif kind == "local":
            off, leaves = _local_cuts(m)
            out = [np.asarray(ctx.check_local_cuts(m.lit_a, m.lit_b, off, leaves)).tolist() for _ in range(2)]
        else:
            raise KeyError(kind)
        q.put((rank, out))
        dist.barrier()
        ctx.close()
    except Exception as e:  # noqa: BLE001
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


def _mp_run(kind, name, world, engine=capi.CEC_ENGINE_AUTO):
    import socket

    import torch.multiprocessing as mp

    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_proc, args=(r, world, port, q, kind, name, engine)) for r in range(world)]
    for p in ps:
        p.start()
    try:
        got = dict(q.get(timeout=300) for _ in ps)
    finally:
        for p in ps:
            p.join(timeout=60)
            if p.is_alive():
                p.kill()
    for r in range(world):
        assert not isinstance(got[r], str), f"rank {r}: {got[r]}"
    return [got[r] for r in range(world)]


@pytest.mark.parametrize("name,world,engine", [
    ("c2bug10", 2, capi.CEC_ENGINE_AUTO),
    ("c5small", 3, capi.CEC_ENGINE_AUTO),
    ("c5small", 2, capi.CEC_ENGINE_INTERP),
    ("tiny", 8, capi.CEC_ENGINE_AUTO),
])
def test_peer_reduction_matches_oracle(name, world, engine):
    """Every rank returns the oracle's per-pair verdict, k and canonical CEX (the global minimum),
    on both calls, and the global CEX vector."""
    m = _workload(name)
    orc = Oracle.from_aig(m.aig)
    ov, oc, ok, _ = orc.check_pairs(m.lit_a, m.lit_b, k_max=32)
    for r, (outs, neq, vecs) in enumerate(_mp_run("sim", name, world, engine)):
        for gv, gc, gk in outs:
            assert_same(np.array(gv), np.array(gc, dtype=np.uint64), np.array(gk), ov, oc, ok,
                        f"{name} world={world} rank={r}")
        for p, vec in zip(neq, vecs):
            assert np.array_equal(np.array(vec), orc.cex_vector(int(m.lit_a[p]), int(m.lit_b[p]), int(oc[p])))


def test_peer_plan_rerun_graph_replay():
    m = _workload("c5small")
    ref = capi.Context.from_aig(m.aig, device=0)
    rv, rc, rk = ref.sim_exhaustive(m.lit_a, m.lit_b)
    neq = rv == capi.CEC_NOT_EQUIVALENT
    assert neq.any()
    for outs in _mp_run("plan", "c5small", 2):
        for gv, gc, gk in outs:
            gv, gc = np.array(gv), np.array(gc, dtype=np.uint64)
            assert np.array_equal(gv, rv) and np.array_equal(np.array(gk), rk)
            assert np.array_equal(gc[neq], rc[neq])


def test_peer_local_checks_match_single():
    """cec_check_local_cuts in peer mode: the same EQ/UNDECIDED verdicts as one GPU."""
    m = _workload("tiny_local")
    off, leaves = _local_cuts(m)
    rv = capi.Context.from_aig(m.aig, device=0).check_local_cuts(m.lit_a, m.lit_b, off, leaves)
    for outs in _mp_run("local", "tiny_local", 2):
        for v in outs:
            assert np.array_equal(np.array(v), rv)


def test_peer_device_barrier_timeout_alone(monkeypatch):
    """The device barrier kernel, run ALONE (no other rank's kernel ever waits on it or is waited
    for): rank 1 of a connected pair never runs, so every barrier of rank 0's run times out after
    CEC_PEER_TIMEOUT_S, sets the error flag, and the call returns CEC_E_NCCL instead of hanging."""
    monkeypatch.setenv("CEC_PEER_TIMEOUT_S", "0.2")
    m = tiny_random(6, 20, 4, 503)
    a = capi.Context.from_aig(m.aig, device=0, rank=0, world=2)
    b = capi.Context.from_aig(m.aig, device=0, rank=1, world=2)
    blobs = [capi.cec_peer_export(a.handle), capi.cec_peer_export(b.handle)]
    capi.cec_peer_import(a.handle, blobs)
    capi.cec_peer_import(b.handle, blobs)
    with pytest.raises(capi.CecError) as ei:
        a.sim_exhaustive(m.lit_a, m.lit_b)
    assert ei.value.status == capi.CEC_E_NCCL


def test_peer_import_rejects_bad_blobs():
    m = tiny_random(6, 20, 4, 503)
    a = capi.Context.from_aig(m.aig, device=0, rank=0, world=2)
    b = capi.Context.from_aig(m.aig, device=0, rank=1, world=2)
    ba, bb = capi.cec_peer_export(a.handle), capi.cec_peer_export(b.handle)
    with pytest.raises(capi.CecError):
        capi.cec_peer_import(a.handle, [bb, ba])  # wrong rank order
    with pytest.raises(capi.CecError):
        capi.cec_peer_import(a.handle, [ba])  # wrong world
    one = capi.Context.from_aig(m.aig, device=0)
    with pytest.raises(capi.CecError):
        capi.cec_peer_export(one.handle)  # world 1: nothing to reduce
