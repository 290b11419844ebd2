"""reduce — TEST INFRASTRUCTURE ONLY (task rule ③). Plain definition of miter reduction.

PAPER.md:61 (§III-A): the miter manager "reduces the miter by merging the proved equivalent pairs";
:185 (§III-D): after each phase "the miter is reduced"; :187: proved pairs are merged and the
fanouts of the non-representative are redirected to the representative (representative = the
minimum id of its class, :41). The merged miter is rebuilt with structural
hashing, as an AIG package does when it re-creates a node (ABC's Aig_And):

    for every AND id in increasing order (a topological order):
        if id is a proved member:  new(id) = new(repr literal)           (fanout redirection)
        else:                      a, b = new(fanin0), new(fanin1), a <= b
                                   a == 0      -> 0          (x & 0)
                                   a == 1      -> b          (x & 1)
                                   a == b      -> a          (x & x)
                                   a == b ^ 1  -> 0          (x & !x)
                                   (a, b) already built -> that node's literal (hash-consing)
                                   else a new AND (a, b) with the next id
    new(0) = 0, new(PI i) = 2 i.

New ids follow creation order, so the result is again in AIGER-binary order. Nothing here is
shared with the product's GPU reduction (csrc/reduce_gpu.cu); only the seeded generators are.
Pins: tests/test_reduce_oracle.py (hand examples, functional equivalence of every node with its
image checked by the independent brute-force evaluator oracle/brute.py, idempotence, identity on a
structurally hashed AIG).
"""
from __future__ import annotations

from typing import Dict, List, Sequence, Tuple


def reduce_miter(num_pis: int, fanins: Sequence[Tuple[int, int]], subst: Dict[int, int],
                 lits: Sequence[int] = ()) -> Tuple[List[Tuple[int, int]], List[int], List[int]]:
    """Returns (new_fanins [(a, b)], image [literal of every old node id in the new AIG], mapped lits).

    subst maps a member AND id to the literal of its representative (whose id is smaller)."""
    A = len(fanins)
    N = 1 + num_pis + A
    image = [0] * N
    for i in range(1, num_pis + 1):
        image[i] = 2 * i
    table: Dict[Tuple[int, int], int] = {}
    out: List[Tuple[int, int]] = []

    def m(lit: int) -> int:
        return image[lit >> 1] ^ (lit & 1)

    for j in range(A):
        nid = 1 + num_pis + j
        if nid in subst:
            r = int(subst[nid])
            if not (r >> 1) < nid:
                raise ValueError(f"representative {r >> 1} of {nid} is not below it")
            image[nid] = m(r)
            continue
        a, b = m(int(fanins[j][0])), m(int(fanins[j][1]))
        if a > b:
            a, b = b, a
        if a == 0:
            image[nid] = 0
        elif a == 1:
            image[nid] = b
        elif a == b:
            image[nid] = a
        elif a == (b ^ 1):
            image[nid] = 0
        elif (a, b) in table:
            image[nid] = table[(a, b)]
        else:
            lit = 2 * (1 + num_pis + len(out))
            out.append((a, b))
            table[(a, b)] = lit
            image[nid] = lit
    return out, image, [m(int(x)) for x in lits]
