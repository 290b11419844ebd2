"""oracle — TEST INFRASTRUCTURE ONLY (task rule ③).

The plain, slow, single-threaded CPU definition of the exhaustive and local checks,
written in C (oracle.c, own AIGER parser) and driven here through ctypes. Only tests/,
__graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may import this package.
It shares no code with paper_conf_dac_liuy25_b200/ and the product never imports it.

The AIG reaches the oracle through an ASCII AIGER file parsed by oracle.c itself, never through the
product's loader.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import tempfile
from typing import Optional, Sequence, Tuple

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
BUILD = os.path.join(HERE, "build")
LIB = os.path.join(BUILD, "liboracle.so")
CLI = os.path.join(BUILD, "oracle")
SRC = [os.path.join(HERE, "oracle.c")]
CLI_SRC = os.path.join(HERE, "oracle_cli.c")

UNDECIDED, EQUIVALENT, NOT_EQUIVALENT, BADCUT = 0, 1, 2, -1
NO_CEX = (1 << 64) - 1


def build(force: bool = False) -> str:
    """Compile liboracle.so and the CLI with plain gcc -O2 (no SIMD flags, single thread)."""
    os.makedirs(BUILD, exist_ok=True)
    newest = max(os.path.getmtime(p) for p in SRC + [CLI_SRC])
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < newest:
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-Wall", "-fPIC", "-shared", "-o", LIB + ".tmp"] + SRC)
        os.replace(LIB + ".tmp", LIB)
    if force or not os.path.exists(CLI) or os.path.getmtime(CLI) < newest:
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-Wall", "-o", CLI + ".tmp", CLI_SRC] + SRC)
        os.replace(CLI + ".tmp", CLI)
    return LIB


_lib = None


def _load():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(LIB)
        P = ctypes.c_void_p
        u32p = ctypes.POINTER(ctypes.c_uint32)
        L.oracle_read_aag.restype = P
        L.oracle_read_aag.argtypes = [ctypes.c_char_p, ctypes.c_char_p, ctypes.c_int]
        L.oracle_free.argtypes = [P]
        for nm in ("oracle_num_pis", "oracle_num_ands", "oracle_num_pos"):
            getattr(L, nm).restype = ctypes.c_uint32
            getattr(L, nm).argtypes = [P]
        L.oracle_support.restype = ctypes.c_int
        L.oracle_support.argtypes = [P, ctypes.c_uint32, ctypes.c_uint32, u32p, ctypes.c_int]
        L.oracle_check_pairs.restype = ctypes.c_uint64
        L.oracle_check_pairs.argtypes = [P, ctypes.c_uint32, P, P, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_uint64,
                                         P, P, P]
        L.oracle_cex_vector.restype = ctypes.c_int
        L.oracle_cex_vector.argtypes = [P, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint64, P]
        L.oracle_eval_lit.restype = ctypes.c_int
        L.oracle_eval_lit.argtypes = [P, ctypes.c_uint32, P]
        L.oracle_eval_all.restype = None
        L.oracle_eval_all.argtypes = [P, P, P]
        L.oracle_check_local.restype = ctypes.c_int
        L.oracle_check_local.argtypes = [P, ctypes.c_uint32, P, P, P, P, P]
        _lib = L
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


class Oracle:
    """An AIG loaded by the oracle's own AIGER parser."""

    def __init__(self, aag_path: str):
        L = _load()
        err = ctypes.create_string_buffer(256)
        self._h = L.oracle_read_aag(aag_path.encode(), err, 256)
        if not self._h:
            raise ValueError(f"oracle: {err.value.decode()}")
        self.num_pis = L.oracle_num_pis(self._h)
        self.num_ands = L.oracle_num_ands(self._h)

    @classmethod
    def from_aig(cls, aig) -> "Oracle":
        """Write `aig` (workloads.Aig) as ASCII AIGER and parse it with the oracle's own reader."""
        from workloads import write_aag  # input generator module (no method arithmetic)
        fd, path = tempfile.mkstemp(suffix=".aag")
        os.close(fd)
        try:
            write_aag(aig, path)
            return cls(path)
        finally:
            os.unlink(path)

    def __del__(self):
        if getattr(self, "_h", None) and _lib is not None:
            _lib.oracle_free(self._h)
            self._h = None

    def support(self, la: int, lb: int) -> list:
        buf = (ctypes.c_uint32 * (self.num_pis + 1))()
        k = _lib.oracle_support(self._h, la, lb, buf, self.num_pis + 1)
        return [int(buf[i]) for i in range(k)]

    def check_pairs(self, lit_a: Sequence[int], lit_b: Sequence[int], k_max: int = 32, lo: int = 0,
                    hi: int = NO_CEX) -> Tuple[np.ndarray, np.ndarray, np.ndarray, int]:
        """Global checks: returns (verdict int32[P], cex uint64[P], k uint32[P], node_evals)."""
        la = np.ascontiguousarray(lit_a, dtype=np.uint32)
        lb = np.ascontiguousarray(lit_b, dtype=np.uint32)
        n = la.size
        v = np.zeros(max(n, 1), dtype=np.int32)
        cex = np.zeros(max(n, 1), dtype=np.uint64)
        k = np.zeros(max(n, 1), dtype=np.uint32)
        ev = _lib.oracle_check_pairs(self._h, n, _ptr(la), _ptr(lb), k_max, lo, hi, _ptr(v), _ptr(cex), _ptr(k))
        return v[:n], cex[:n], k[:n], int(ev)

    def cex_vector(self, la: int, lb: int, idx: int) -> np.ndarray:
        out = np.zeros(max(self.num_pis, 1), dtype=np.uint8)
        _lib.oracle_cex_vector(self._h, la, lb, idx, _ptr(out))
        return out[:self.num_pis]

    def eval_lit(self, lit: int, pis: np.ndarray) -> int:
        p = np.ascontiguousarray(pis, dtype=np.uint8)
        return int(_lib.oracle_eval_lit(self._h, lit, _ptr(p)))

    def eval_all(self, pis: np.ndarray) -> np.ndarray:
        """Value (0/1) of every node id under one PI assignment (PI id i+1 = pis[i])."""
        p = np.ascontiguousarray(pis, dtype=np.uint8)
        out = np.zeros(1 + self.num_pis + self.num_ands, dtype=np.uint8)
        _lib.oracle_eval_all(self._h, _ptr(p), _ptr(out))
        return out

    def check_local(self, lit_a, lit_b, cut_off, leaves) -> np.ndarray:
        la = np.ascontiguousarray(lit_a, dtype=np.uint32)
        lb = np.ascontiguousarray(lit_b, dtype=np.uint32)
        off = np.ascontiguousarray(cut_off, dtype=np.uint32)
        lv = np.ascontiguousarray(leaves if len(leaves) else [0], dtype=np.uint32)
        v = np.zeros(max(la.size, 1), dtype=np.int32)
        _lib.oracle_check_local(self._h, la.size, _ptr(la), _ptr(lb), _ptr(off), _ptr(lv), _ptr(v))
        return v[:la.size]


def run_cli(*args: str) -> str:
    build()
    return subprocess.check_output([CLI, *args], text=True)
