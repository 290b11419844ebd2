"""Thin ctypes binding of include/cec.h (argument marshalling only; every step of the hot path runs
in libcec.so's sm_100a kernels and its C++ host driver). Function names match the C ABI.

There is no fallback: if libcec.so is missing this module raises ImportError, and on a machine
without a CUDA device every simulation call raises CecError(CEC_E_CUDA).
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional, Sequence, Tuple

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libcec.so")

CEC_OK, CEC_E_ARG, CEC_E_AIG, CEC_E_CUT, CEC_E_NOMEM, CEC_E_CUDA, CEC_E_NCCL, CEC_E_NOCEX, CEC_E_STATE = range(9)
CEC_BAD_CUT, CEC_UNDECIDED, CEC_EQUIVALENT, CEC_NOT_EQUIVALENT = -1, 0, 1, 2
CEC_MERGE_OFF, CEC_MERGE_PAPER, CEC_MERGE_COST = 0, 1, 2
CEC_ENGINE_AUTO, CEC_ENGINE_INTERP, CEC_ENGINE_JIT, CEC_ENGINE_SIMT = 0, 1, 2, 3
CEC_NO_CEX = (1 << 64) - 1
STATUS_NAMES = ["CEC_OK", "CEC_E_ARG", "CEC_E_AIG", "CEC_E_CUT", "CEC_E_NOMEM", "CEC_E_CUDA", "CEC_E_NCCL",
                "CEC_E_NOCEX", "CEC_E_STATE"]

# every symbol include/cec.h declares (tests check the library exports all of them)
EXPORTS = ["cec_default_opts", "cec_load_aig", "cec_sim_exhaustive", "cec_check_local_cuts", "cec_get_cex",
           "cec_pair_support", "cec_plan_exhaustive", "cec_plan_run", "cec_plan_results", "cec_plan_info",
           "cec_plan_window", "cec_plan_free", "cec_stream", "cec_get_stats", "cec_shard_range", "cec_pext64",
           "cec_free", "cec_last_error", "cec_abi_version", "cec_nccl_unique_id", "cec_sim_random",
           "cec_common_cuts", "cec_sim_patterns", "cec_reduce", "cec_sim_classes", "cec_local_pass",
           "cec_peer_export", "cec_peer_import", "cec_peer_host_barrier", "cec_reload_aig", "cec_plan_sweep_ms",
           "cec_plan_sweep_timing"]


class CecOpts(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int32), ("rank", ctypes.c_int32), ("world", ctypes.c_int32),
                ("nccl_unique_id", ctypes.c_void_p), ("stream", ctypes.c_void_p), ("k_max", ctypes.c_uint32),
                ("k_s", ctypes.c_uint32), ("merge", ctypes.c_int32), ("engine", ctypes.c_int32),
                ("workspace", ctypes.c_void_p), ("workspace_bytes", ctypes.c_uint64), ("reserved", ctypes.c_uint64 * 4)]


class CecAig(ctypes.Structure):
    _fields_ = [("num_pis", ctypes.c_uint32), ("num_ands", ctypes.c_uint32), ("num_pos", ctypes.c_uint32),
                ("fanin_lits", ctypes.c_void_p), ("po_lits", ctypes.c_void_p)]


class CecStats(ctypes.Structure):
    _fields_ = [("node_patterns", ctypes.c_uint64), ("node_patterns_all", ctypes.c_uint64),
                ("num_windows", ctypes.c_uint32), ("max_k", ctypes.c_uint32), ("max_slots", ctypes.c_uint32),
                ("num_launches", ctypes.c_uint32), ("kernel_ms", ctypes.c_float), ("host_prep_ms", ctypes.c_float),
                ("h2d_bytes", ctypes.c_uint64), ("d2h_bytes", ctypes.c_uint64), ("jit_ms", ctypes.c_float),
                ("jit_kernels", ctypes.c_uint32), ("jit_windows", ctypes.c_uint32), ("lop3_words", ctypes.c_uint64),
                ("imad_words", ctypes.c_uint64)]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


class CecError(RuntimeError):
    def __init__(self, status: int, msg: str):
        self.status = status
        super().__init__(f"{STATUS_NAMES[status] if 0 <= status < len(STATUS_NAMES) else status}: {msg}")


def _load() -> ctypes.CDLL:
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: run `python -c 'import __graft_entry__ as g; g.build()'` "
                          "(there is no CPU fallback)")
    L = ctypes.CDLL(LIB_PATH)
    P, u32, u64, i32 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int32
    sig = {
        "cec_default_opts": (None, [P]),
        "cec_load_aig": (ctypes.c_int, [P, P, P]),
        "cec_reload_aig": (ctypes.c_int, [P, P, ctypes.c_uint32, ctypes.c_uint32]),
        "cec_plan_sweep_ms": (ctypes.c_int, [P, P]),
        "cec_plan_sweep_timing": (ctypes.c_int, [P, ctypes.c_int]),
        "cec_sim_exhaustive": (ctypes.c_int, [P, u32, P, P, P, P, P]),
        "cec_check_local_cuts": (ctypes.c_int, [P, u32, P, P, P, P, P]),
        "cec_get_cex": (ctypes.c_int, [P, u32, P]),
        "cec_pair_support": (ctypes.c_int, [P, u32, u32, P, u32, P]),
        "cec_plan_exhaustive": (ctypes.c_int, [P, u32, P, P, P]),
        "cec_plan_run": (ctypes.c_int, [P, P]),
        "cec_plan_results": (ctypes.c_int, [P, P, P, P, P]),
        "cec_plan_info": (ctypes.c_int, [P, P, P, P, P]),
        "cec_plan_window": (ctypes.c_int, [P, u32, P, P, P, P, P]),
        "cec_plan_free": (None, [P]),
        "cec_stream": (P, [P]),
        "cec_get_stats": (ctypes.c_int, [P, P]),
        "cec_shard_range": (None, [u64, i32, i32, P, P]),
        "cec_pext64": (u64, [u64, u64]),
        "cec_free": (None, [P]),
        "cec_last_error": (ctypes.c_char_p, [P]),
        "cec_abi_version": (ctypes.c_int, []),
        "cec_nccl_unique_id": (ctypes.c_int, [P]),
        "cec_peer_export": (ctypes.c_int, [P, P]),
        "cec_peer_import": (ctypes.c_int, [P, P]),
        "cec_peer_host_barrier": (ctypes.c_int, [P, P, P]),
        "cec_sim_random": (ctypes.c_int, [P, u32, u64, P, P]),
        "cec_common_cuts": (ctypes.c_int, [P, u32, P, P, u32, u32, i32, u32, P, P, P]),
        "cec_sim_patterns": (ctypes.c_int, [P, u32, P, P, P]),
        "cec_reduce": (ctypes.c_int, [P, u32, P, P, P, P, P, u32, P]),
        "cec_sim_classes": (ctypes.c_int, [P, u32, u64, u32, P, u32, P, P, P, P]),
        "cec_local_pass": (ctypes.c_int, [P, u32, P, P, P, u32, u32, i32, u32, u32, P, P, P, P, P, P]),
    }
    for name, (res, args) in sig.items():
        fn = getattr(L, name)
        fn.restype = res
        fn.argtypes = args
    return L


lib = _load()


def _p(a: Optional[np.ndarray]):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _u32(x) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(x, dtype=np.uint32).reshape(-1))


def cec_default_opts(**kw) -> CecOpts:
    o = CecOpts()
    lib.cec_default_opts(ctypes.byref(o))
    for k, v in kw.items():
        setattr(o, k, v)
    return o


def cec_last_error(ctx) -> str:
    s = lib.cec_last_error(ctx)
    return s.decode(errors="replace") if s else ""


def _check(st: int, ctx=None):
    if st != CEC_OK:
        raise CecError(st, cec_last_error(ctx))


def cec_load_aig(num_pis: int, fanins: np.ndarray, pos: np.ndarray, opts: Optional[CecOpts] = None,
                 nccl_unique_id: Optional[bytes] = None):
    fan = _u32(fanins)
    po = _u32(pos)
    aig = CecAig(num_pis, fan.size // 2, po.size, fan.ctypes.data if fan.size else None,
                 po.ctypes.data if po.size else None)
    opts = opts if opts is not None else cec_default_opts()
    keep = None
    if nccl_unique_id is not None:
        keep = ctypes.create_string_buffer(bytes(nccl_unique_id), 128)
        opts.nccl_unique_id = ctypes.cast(keep, ctypes.c_void_p)
    ctx = ctypes.c_void_p()
    st = lib.cec_load_aig(ctypes.byref(ctx), ctypes.byref(aig), ctypes.byref(opts))
    _check(st, None)
    return ctx


def cec_reload_aig(ctx, num_pis: int, fanins: np.ndarray, pos: np.ndarray, k_max: int = 0, k_s: int = 0) -> None:
    """Next miter version into the same context (include/cec.h cec_reload_aig; 0 = keep the limit)."""
    fan = _u32(fanins)
    po = _u32(pos)
    aig = CecAig(num_pis, fan.size // 2, po.size, fan.ctypes.data if fan.size else None,
                 po.ctypes.data if po.size else None)
    _check(lib.cec_reload_aig(ctx, ctypes.byref(aig), int(k_max), int(k_s)), ctx)


def cec_free(ctx) -> None:
    lib.cec_free(ctx)


def _pair_arrays(lit_a, lit_b) -> Tuple[np.ndarray, np.ndarray]:
    """Both sides of a pair list as uint32 arrays of ONE length: the C side reads num_pairs entries
    of each, so a shorter buffer would be read past its end."""
    la, lb = _u32(lit_a), _u32(lit_b)
    if la.size != lb.size:
        raise ValueError(f"lit_a has {la.size} entries, lit_b {lb.size}")
    return la, lb


def _ids_arrays(*arrs) -> Tuple[np.ndarray, ...]:
    out = tuple(_u32(a) for a in arrs)
    if len({a.size for a in out}) > 1:
        raise ValueError(f"per-pair arrays differ in length: {[a.size for a in out]}")
    return out


def cec_sim_exhaustive(ctx, lit_a, lit_b) -> Tuple[np.ndarray, np.ndarray, np.ndarray]:
    la, lb = _pair_arrays(lit_a, lit_b)
    n = la.size
    v = np.zeros(max(n, 1), np.int32)
    cex = np.zeros(max(n, 1), np.uint64)
    k = np.zeros(max(n, 1), np.uint32)
    _check(lib.cec_sim_exhaustive(ctx, n, _p(la), _p(lb), _p(v), _p(cex), _p(k)), ctx)
    return v[:n], cex[:n], k[:n]


def cec_check_local_cuts(ctx, lit_a, lit_b, cut_off, cut_leaves, raise_on_bad_cut: bool = False) -> np.ndarray:
    la, lb = _pair_arrays(lit_a, lit_b)
    off = _u32(cut_off)
    n = la.size
    nl = len(cut_leaves)
    # CSR cut_off[n+1] (include/cec.h): the C side reads cut_leaves[cut_off[i] .. cut_off[i+1])
    if off.size != n + 1 or int(off[0]) != 0 or int(off[-1]) != nl or (n and np.any(np.diff(off.astype(np.int64)) < 0)):
        raise ValueError(f"cut_off must be a non-decreasing CSR offset array of {n + 1} entries from 0 to {nl}")
    lv = _u32(cut_leaves) if nl else np.zeros(1, np.uint32)
    v = np.zeros(max(n, 1), np.int32)
    st = lib.cec_check_local_cuts(ctx, n, _p(la), _p(lb), _p(off), _p(lv), _p(v))
    if st == CEC_E_CUT and not raise_on_bad_cut:
        return v[:n]
    _check(st, ctx)
    return v[:n]


def cec_sim_random(ctx, num_nodes: int, num_words: int = 64, seed: int = 1):
    """Per-node complement-canonical random-simulation signatures (uint64[N]) and phases (uint8[N])."""
    sig = np.zeros(max(num_nodes, 1), np.uint64)
    ph = np.zeros(max(num_nodes, 1), np.uint8)
    _check(lib.cec_sim_random(ctx, num_words, seed, _p(sig), _p(ph)), ctx)
    return sig[:num_nodes], ph[:num_nodes]


def cec_sim_patterns(ctx, num_nodes: int, pi_words: np.ndarray):
    """Signatures for caller patterns: pi_words uint32 [num_pis, num_words] (PI id i+1 = row i)."""
    w = np.ascontiguousarray(pi_words, dtype=np.uint32)
    sig = np.zeros(max(num_nodes, 1), np.uint64)
    ph = np.zeros(max(num_nodes, 1), np.uint8)
    _check(lib.cec_sim_patterns(ctx, w.shape[1], _p(w), _p(sig), _p(ph)), ctx)
    return sig[:num_nodes], ph[:num_nodes]


def cec_common_cuts(ctx, repr_ids, member_ids, k_l: int, C: int, pass_id: int, max_cuts: int):
    """Common cuts per candidate pair: (pair_cut_off[n+1], cut_off[ncut+1], leaves[...])."""
    r, m = _ids_arrays(repr_ids, member_ids)
    n = r.size
    pco = np.zeros(n + 1, np.uint32)
    co = np.zeros(n * max_cuts + 1, np.uint32)
    lv = np.zeros(max(1, n * max_cuts * k_l), np.uint32)
    _check(lib.cec_common_cuts(ctx, n, _p(r), _p(m), k_l, C, pass_id, max_cuts, _p(pco), _p(co), _p(lv)), ctx)
    ncut = int(pco[n])
    return pco, co[:ncut + 1], lv[:int(co[ncut])]


def cec_sim_classes(ctx, num_words: int, seed: int, pi_words: Optional[np.ndarray] = None, cap: Optional[int] = None):
    """GPU equivalence classes: (repr uint32[P], member uint32[P], phase uint8[P]) ordered by member.
    pi_words: optional uint32 [num_pis, Wc] caller patterns (PI id i+1 = row i)."""
    w = None if pi_words is None else np.ascontiguousarray(pi_words, dtype=np.uint32)
    wc = 0 if w is None else int(w.shape[1])
    total = ctypes.c_uint32()
    if cap is None:  # ask for the count first, then fetch
        _check(lib.cec_sim_classes(ctx, num_words, seed, wc, _p(w), 0, ctypes.byref(total), None, None, None), ctx)
        cap = int(total.value)
    r = np.zeros(max(cap, 1), np.uint32)
    m = np.zeros(max(cap, 1), np.uint32)
    ph = np.zeros(max(cap, 1), np.uint8)
    _check(lib.cec_sim_classes(ctx, num_words, seed, wc, _p(w), cap, ctypes.byref(total), _p(r), _p(m), _p(ph)), ctx)
    n = min(cap, int(total.value))
    return r[:n], m[:n], ph[:n]


def cec_reduce(ctx, num_pis: int, num_ands: int, member_ids, repr_lits, lits=()):
    """GPU miter reduction: returns (new_fanins uint32 [A', 2], image uint32 [N], mapped lits)."""
    m, r = _ids_arrays(member_ids, repr_lits)
    lv = _u32(lits).copy()
    fan = np.zeros(max(2 * num_ands, 2), np.uint32)
    img = np.zeros(1 + num_pis + num_ands, np.uint32)
    na = ctypes.c_uint32()
    _check(lib.cec_reduce(ctx, m.size, _p(m), _p(r), ctypes.byref(na), _p(fan), _p(img), lv.size,
                          _p(lv) if lv.size else None), ctx)
    return fan[:2 * na.value].reshape(-1, 2), img, lv


def cec_local_pass(ctx, repr_ids, member_ids, phases, k_l: int, C: int, pass_id: int, max_cuts: int,
                   buffer_checks: int = 4096, log: bool = True):
    """Alg. 2 pass: (verdict int32[npairs], checks) where checks = (pair uint32[n], cut_off uint32[n+1],
    leaves uint32[...], verdict int32[n]) in issue order (None when log=False)."""
    r, m = _ids_arrays(repr_ids, member_ids)
    ph = np.ascontiguousarray(np.asarray(phases, dtype=np.uint8).reshape(-1))
    if ph.size != r.size:
        raise ValueError(f"phases has {ph.size} entries, expected {r.size}")
    n = r.size
    v = np.zeros(max(n, 1), np.int32)
    nc = ctypes.c_uint32()
    cap = max(1, n * max_cuts)
    cp = np.zeros(cap, np.uint32) if log else None
    co = np.zeros(cap + 1, np.uint32) if log else None
    cl = np.zeros(max(1, cap * k_l), np.uint32) if log else None
    cv = np.zeros(cap, np.int32) if log else None
    _check(lib.cec_local_pass(ctx, n, _p(r), _p(m), _p(ph), k_l, C, pass_id, max_cuts, buffer_checks, _p(v),
                              ctypes.byref(nc), _p(cp), _p(co), _p(cl), _p(cv)), ctx)
    k = int(nc.value)
    checks = (cp[:k], co[:k + 1], cl[:int(co[k])], cv[:k]) if log else None
    return v[:n], checks


def cec_get_cex(ctx, pair_idx: int, num_pis: int) -> np.ndarray:
    out = np.zeros(max(num_pis, 1), np.uint8)
    _check(lib.cec_get_cex(ctx, pair_idx, _p(out)), ctx)
    return out[:num_pis]


def cec_pair_support(ctx, lit_a: int, lit_b: int) -> list:
    """Full structural support (sorted PI ids) of {var(lit_a), var(lit_b)}."""
    k = cec_pair_k(ctx, lit_a, lit_b)
    buf = np.zeros(max(k, 1), np.uint32)
    kk = ctypes.c_uint32()
    _check(lib.cec_pair_support(ctx, lit_a, lit_b, _p(buf), k, ctypes.byref(kk)), ctx)
    return [int(x) for x in buf[:k]]


def cec_pair_k(ctx, lit_a: int, lit_b: int) -> int:
    k = ctypes.c_uint32()
    _check(lib.cec_pair_support(ctx, lit_a, lit_b, None, 0, ctypes.byref(k)), ctx)
    return int(k.value)


def cec_plan_exhaustive(ctx, lit_a, lit_b):
    la, lb = _pair_arrays(lit_a, lit_b)
    plan = ctypes.c_void_p()
    _check(lib.cec_plan_exhaustive(ctx, la.size, _p(la), _p(lb), ctypes.byref(plan)), ctx)
    return plan


def cec_plan_run(ctx, plan) -> None:
    _check(lib.cec_plan_run(ctx, plan), ctx)


def cec_plan_results(ctx, plan, num_pairs: int):
    v = np.zeros(max(num_pairs, 1), np.int32)
    cex = np.zeros(max(num_pairs, 1), np.uint64)
    k = np.zeros(max(num_pairs, 1), np.uint32)
    _check(lib.cec_plan_results(ctx, plan, _p(v), _p(cex), _p(k)), ctx)
    return v[:num_pairs], cex[:num_pairs], k[:num_pairs]


def cec_plan_sweep_timing(plan, on: bool) -> None:
    """Record (or stop recording) the window-kernel events in the plan's runs (include/cec.h)."""
    _check(lib.cec_plan_sweep_timing(plan, 1 if on else 0), None)


def cec_plan_sweep_ms(plan) -> float:
    """Window-kernel device time of the plan's last completed run (include/cec.h); sync first."""
    ms = ctypes.c_float()
    _check(lib.cec_plan_sweep_ms(plan, ctypes.byref(ms)), None)
    return float(ms.value)


def cec_plan_info(plan) -> dict:
    nw, W, mk, ms = ctypes.c_uint32(), ctypes.c_uint64(), ctypes.c_uint32(), ctypes.c_uint32()
    _check(lib.cec_plan_info(plan, ctypes.byref(nw), ctypes.byref(W), ctypes.byref(mk), ctypes.byref(ms)))
    return {"num_windows": nw.value, "node_patterns": W.value, "max_k": mk.value, "max_slots": ms.value}


def cec_plan_window(plan, w: int) -> dict:
    k, nn, np_ = ctypes.c_uint32(), ctypes.c_uint32(), ctypes.c_uint32()
    _check(lib.cec_plan_window(plan, w, None, ctypes.byref(k), ctypes.byref(nn), None, ctypes.byref(np_)))
    ins = np.zeros(max(k.value, 1), np.uint32)
    pairs = np.zeros(max(np_.value, 1), np.uint32)
    _check(lib.cec_plan_window(plan, w, _p(ins), None, None, _p(pairs), None))
    return {"inputs": [int(x) for x in ins[:k.value]], "num_nodes": nn.value,
            "pairs": [int(x) for x in pairs[:np_.value]]}


def cec_plan_free(plan) -> None:
    lib.cec_plan_free(plan)


def cec_stream(ctx) -> int:
    return lib.cec_stream(ctx) or 0


def cec_get_stats(ctx) -> dict:
    s = CecStats()
    _check(lib.cec_get_stats(ctx, ctypes.byref(s)), ctx)
    return s.as_dict()


def cec_shard_range(n: int, rank: int, world: int) -> Tuple[int, int]:
    b, e = ctypes.c_uint64(), ctypes.c_uint64()
    lib.cec_shard_range(n, rank, world, ctypes.byref(b), ctypes.byref(e))
    return b.value, e.value


def cec_pext64(value: int, mask: int) -> int:
    return int(lib.cec_pext64(value, mask))


def cec_nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(lib.cec_nccl_unique_id(buf), None)
    return buf.raw


PEER_BLOB_BYTES = 128


def cec_peer_export(ctx) -> bytes:
    """This rank's exchange-block blob (CUDA IPC handle + pid/device/rank), include/cec.h."""
    buf = ctypes.create_string_buffer(PEER_BLOB_BYTES)
    _check(lib.cec_peer_export(ctx, buf), ctx)
    return buf.raw


def cec_peer_import(ctx, blobs) -> None:
    """Map every rank's exchange block (blobs in rank order) and switch the context to peer mode."""
    raw = b"".join(bytes(b) for b in blobs)
    if len(raw) != PEER_BLOB_BYTES * len(blobs):
        raise ValueError("peer blobs must be 128 bytes each")
    _check(lib.cec_peer_import(ctx, ctypes.create_string_buffer(raw, len(raw))), ctx)


HOST_BARRIER_FN = ctypes.CFUNCTYPE(None, ctypes.c_void_p)


def cec_peer_host_barrier(ctx, fn) -> object:
    """Several ranks emulated on ONE device (tests): every peer barrier becomes "drain the stream,
    then fn()" (include/cec.h cec_peer_host_barrier). Returns the ctypes callback, which the caller
    keeps alive as long as the context uses it; fn = None restores the device barriers."""
    cb = HOST_BARRIER_FN(lambda _user: fn()) if fn is not None else None
    _check(lib.cec_peer_host_barrier(ctx, ctypes.cast(cb, ctypes.c_void_p) if cb else None, None), ctx)
    return cb


def cec_abi_version() -> int:
    return int(lib.cec_abi_version())


class Context:
    """RAII wrapper around a cec_ctx for one AIG."""

    def __init__(self, num_pis: int, fanins: np.ndarray, pos: np.ndarray, **opt):
        uid = opt.pop("nccl_unique_id", None)
        self.opts = cec_default_opts(**opt)
        self.num_pis = num_pis
        self.num_ands = int(np.asarray(fanins).reshape(-1, 2).shape[0])
        self._ctx = cec_load_aig(num_pis, fanins, pos, self.opts, nccl_unique_id=uid)

    @classmethod
    def from_aig(cls, aig, **opt) -> "Context":
        return cls(aig.num_pis, aig.fanins, aig.pos, **opt)

    @property
    def handle(self):
        return self._ctx

    def reload(self, aig, k_max: int = 0, k_s: int = 0) -> "Context":
        """Replace the AIG (the next miter version), keeping streams, workers, pools and JIT kernels."""
        cec_reload_aig(self._ctx, aig.num_pis, aig.fanins, aig.pos, k_max, k_s)
        self.num_pis = aig.num_pis
        self.num_ands = int(aig.num_ands)
        return self

    def sim_exhaustive(self, lit_a, lit_b):
        return cec_sim_exhaustive(self._ctx, lit_a, lit_b)

    def check_local_cuts(self, lit_a, lit_b, cut_off, leaves):
        return cec_check_local_cuts(self._ctx, lit_a, lit_b, cut_off, leaves)

    def get_cex(self, pair_idx: int) -> np.ndarray:
        return cec_get_cex(self._ctx, pair_idx, self.num_pis)

    def sim_classes(self, num_words: int, seed: int, pi_words=None, cap=None):
        # every member is an AND node, so num_ands bounds the pair count: one call, no count pass
        return cec_sim_classes(self._ctx, num_words, seed, pi_words, max(1, self.num_ands) if cap is None else cap)

    def reduce(self, member_ids, repr_lits, lits=()):
        return cec_reduce(self._ctx, self.num_pis, self.num_ands, member_ids, repr_lits, lits)

    def peer_connect(self, all_gather, host_barrier=None) -> None:
        """Peer-memory a10 (include/cec.h cec_peer_export/import): `all_gather(blob) -> [blob of
        rank 0, ..., rank world-1]` is the caller's collective (e.g. torch.distributed
        all_gather_object); every rank calls this once, collectively. `host_barrier` (ranks
        emulated on one device only): the callable that replaces the device barriers."""
        cec_peer_import(self._ctx, all_gather(cec_peer_export(self._ctx)))
        if host_barrier is not None:
            self._host_barrier_cb = cec_peer_host_barrier(self._ctx, host_barrier)

    def pair_k(self, lit_a: int, lit_b: int) -> int:
        return cec_pair_k(self._ctx, lit_a, lit_b)

    def stats(self) -> dict:
        return cec_get_stats(self._ctx)

    def close(self):
        if getattr(self, "_ctx", None):
            cec_free(self._ctx)
            self._ctx = None

    def __del__(self):
        try:
            self.close()
        except TypeError:  # interpreter shutdown: module globals already torn down
            pass
