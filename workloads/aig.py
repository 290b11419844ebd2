"""AIG container, structural builder and AIGER (ASCII) I/O for the seeded workload generators.

This module is *input generation only*: it builds graphs and writes/reads files. It holds none of the
method's arithmetic (no simulation, no truth tables, no supports, no comparison), so both the CUDA
path and the oracle may consume what it produces.

Conventions (§II-A "AIG"):
  * node id 0 = constant 0, ids 1..I = PIs in input order, ids I+1..I+A = AND nodes;
  * a literal is 2*id + complement;
  * every AND's fanin ids are smaller than its own id (AIGER-binary order), so id order is a
    topological order.
"""
from __future__ import annotations

import dataclasses
import os
from typing import Dict, Iterable, List, Optional, Sequence, Tuple

import numpy as np


@dataclasses.dataclass
class Aig:
    num_pis: int
    fanins: np.ndarray  # uint32 [A, 2] AIGER literals
    pos: np.ndarray  # uint32 [O] AIGER literals

    @property
    def num_ands(self) -> int:
        return int(self.fanins.shape[0])

    @property
    def num_nodes(self) -> int:
        return 1 + self.num_pis + self.num_ands

    def validate(self) -> None:
        I = self.num_pis
        A = self.num_ands
        if self.fanins.dtype != np.uint32 or self.pos.dtype != np.uint32:
            raise ValueError("arrays must be uint32")
        if A:
            own = (1 + I + np.arange(A, dtype=np.int64))[:, None]
            ids = self.fanins.astype(np.int64) >> 1
            if not np.all(ids < own):
                raise ValueError("fanin id not below own id")
        if self.pos.size and int(self.pos.max()) >> 1 >= 1 + I + A:
            raise ValueError("PO literal out of range")


class Builder:
    """Structural AIG builder with optional structural hashing (strash).

    Only graph construction lives here (constant folding of AND(x,0), AND(x,x), AND(x,!x) and
    hash-consing are structural rules, not simulation)."""

    def __init__(self, num_pis: int, strash: bool = True):
        self.num_pis = num_pis
        self.ands: List[Tuple[int, int]] = []
        self.strash = strash
        self._table: Dict[Tuple[int, int], int] = {}

    # -- literals ------------------------------------------------------------------------------
    def pi(self, i: int) -> int:
        if not 0 <= i < self.num_pis:
            raise IndexError(i)
        return 2 * (1 + i)

    def next_id(self) -> int:
        return 1 + self.num_pis + len(self.ands)

    def AND(self, a: int, b: int) -> int:
        if a > b:
            a, b = b, a
        if a == 0:
            return 0
        if a == 1:
            return b
        if a == b:
            return a
        if a == (b ^ 1):
            return 0
        if self.strash:
            key = (a, b)
            hit = self._table.get(key)
            if hit is not None:
                return hit
        lit = 2 * self.next_id()
        self.ands.append((a, b))
        if self.strash:
            self._table[(a, b)] = lit
        return lit

    def raw_and(self, a: int, b: int) -> int:
        """Append an AND without folding or hashing (used to force distinct structure)."""
        lit = 2 * self.next_id()
        self.ands.append((a, b))
        return lit

    def OR(self, a: int, b: int) -> int:
        return self.AND(a ^ 1, b ^ 1) ^ 1

    def XOR(self, a: int, b: int) -> int:
        # (a & !b) | (!a & b): 3 ANDs
        return self.OR(self.AND(a, b ^ 1), self.AND(a ^ 1, b))

    def XOR_alt(self, a: int, b: int) -> int:
        # (a | b) & !(a & b): the other 3-AND XOR form (SURVEY.md §8(d) "alternative XOR forms")
        return self.AND(self.OR(a, b), self.AND(a, b) ^ 1)

    def MUX(self, s: int, t: int, e: int) -> int:
        return self.OR(self.AND(s, t), self.AND(s ^ 1, e))

    def MAJ(self, a: int, b: int, c: int) -> int:
        return self.OR(self.AND(a, b), self.AND(c, self.OR(a, b)))

    def MAJ_alt(self, a: int, b: int, c: int) -> int:
        return self.OR(self.OR(self.AND(a, b), self.AND(a, c)), self.AND(b, c))

    def finish(self, pos: Sequence[int]) -> Aig:
        fan = np.asarray(self.ands, dtype=np.uint32).reshape(-1, 2)
        aig = Aig(self.num_pis, fan, np.asarray(list(pos), dtype=np.uint32))
        aig.validate()
        return aig


# ---------------------------------------------------------------------------------------------
# AIGER ASCII I/O
# ---------------------------------------------------------------------------------------------

def write_aag(aig: Aig, path: str) -> None:
    I, A, O = aig.num_pis, aig.num_ands, int(aig.pos.size)
    M = I + A
    lines = [f"aag {M} {I} 0 {O} {A}"]
    lines += [str(2 * (1 + i)) for i in range(I)]
    lines += [str(int(p)) for p in aig.pos]
    lhs = 2 * (1 + I + np.arange(A, dtype=np.int64))
    f = aig.fanins.astype(np.int64)
    # AIGER requires rhs0 >= rhs1 only in the binary format; ASCII accepts any order
    lines += [f"{int(l)} {int(a)} {int(b)}" for l, a, b in zip(lhs, f[:, 0], f[:, 1])]
    tmp = path + ".tmp"
    with open(tmp, "w") as fh:
        fh.write("\n".join(lines) + "\n")
    os.replace(tmp, path)


def read_aag(path: str) -> Aig:
    """Read an ASCII AIGER file and renumber it into AIGER-binary order:
    PIs keep their input order as ids 1..I; ANDs are renumbered in a topological order that keeps
    the file order whenever it is already topological. Latches are rejected (combinational only)."""
    with open(path) as fh:
        tok = fh.read().split("\n")
    hdr = tok[0].split()
    if hdr[0] != "aag":
        raise ValueError("not an ASCII AIGER file")
    M, I, L, O, A = (int(x) for x in hdr[1:6])
    if L != 0:
        raise ValueError("latches are not supported (combinational CEC only)")
    p = 1
    in_lits = [int(tok[p + i]) for i in range(I)]
    p += I
    out_lits = [int(tok[p + i]) for i in range(O)]
    p += O
    gates = []
    for i in range(A):
        a, b, c = (int(x) for x in tok[p + i].split()[:3])
        gates.append((a, b, c))
    var_map = {0: 0}
    for i, l in enumerate(in_lits):
        var_map[l >> 1] = 1 + i
    by_var = {g[0] >> 1: g for g in gates}
    order: List[int] = []
    state: Dict[int, int] = {}
    for g in gates:  # iterative DFS to get a topological order
        stack = [(g[0] >> 1, 0)]
        while stack:
            v, st = stack.pop()
            if v in var_map or state.get(v) == 2:
                continue
            if st == 0:
                if state.get(v) == 1:
                    raise ValueError("combinational cycle")
                state[v] = 1
                stack.append((v, 1))
                gg = by_var[v]
                for f in (gg[2] >> 1, gg[1] >> 1):
                    if f not in var_map and state.get(f) != 2:
                        if f not in by_var:
                            raise ValueError(f"undefined variable {f}")
                        stack.append((f, 0))
            else:
                state[v] = 2
                var_map[v] = 1 + I + len(order)
                order.append(v)

    def ml(l: int) -> int:
        return 2 * var_map[l >> 1] + (l & 1)

    fan = np.array([(ml(by_var[v][1]), ml(by_var[v][2])) for v in order], dtype=np.uint32).reshape(-1, 2)
    aig = Aig(I, fan, np.array([ml(l) for l in out_lits], dtype=np.uint32))
    aig.validate()
    return aig


def write_pairs(path: str, lit_a: Iterable[int], lit_b: Iterable[int]) -> None:
    la, lb = list(lit_a), list(lit_b)
    with open(path, "w") as fh:
        fh.write(f"{len(la)}\n")
        for a, b in zip(la, lb):
            fh.write(f"{a} {b}\n")


def write_checks(path: str, lit_a, lit_b, cut_off, leaves) -> None:
    with open(path, "w") as fh:
        fh.write(f"{len(lit_a)}\n")
        for q in range(len(lit_a)):
            lv = leaves[cut_off[q]:cut_off[q + 1]]
            fh.write(" ".join(str(int(x)) for x in [lit_a[q], lit_b[q], len(lv), *lv]) + "\n")
