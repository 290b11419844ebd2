"""cuts — TEST INFRASTRUCTURE ONLY. Plain-Python definition of the cut generator used for local
function checking (§III-C1, :132-154), written set by set so it can be read against the
paper. The product's generators (csrc/cuts.cpp on the host; any GPU version) must return exactly
these cuts. Exact arithmetic throughout (Fractions), so tie-breaking is unambiguous.

Definition (with the readings fixed in DESIGN.md):
  * E(n) = { u ∪ v : u ∈ P(n0) ∪ {{n0}}, v ∈ P(n1) ∪ {{n1}}, |u ∪ v| ≤ k_l }       (Eq. 1)
    minus the empty set and {n}; the constant node contributes no leaf ({0} is the empty set).
  * dominated cuts (a proper superset of another cut of E(n)) are dropped (priority cuts [27]).
  * ranking (Table I), pass 0: larger mean fanout, smaller size, smaller mean level;
    pass 1: smaller mean level, smaller size, larger mean fanout; pass 2: larger mean level,
    smaller size, larger mean fanout; remaining ties: lexicographic order of the sorted leaf list.
  * a non-representative n (repr_of[n] = r) ranks first by larger similarity
    s(c, P(r)) = Σ_{c' ∈ P(r)} |c ∩ c'| / |c ∪ c'|, then as above.
  * P(n) = the first C; PIs have P = {{pi}} (Alg. 2 l.4-5). Nodes are visited in increasing id.
  * common cuts of a pair (r, m): { u ∪ v : u ∈ P(r), v ∈ P(m), |u ∪ v| ≤ k_l }, non-empty, sorted by
    (size, lexicographic), the first max_cuts.
Only nodes in the transitive fanin of the pairs are enumerated (others cannot matter).
"""
from __future__ import annotations

from fractions import Fraction
from typing import Dict, List, Sequence, Tuple


def _tfi(num_pis: int, fanins, roots) -> set:
    seen, todo = set(), list(roots)
    while todo:
        v = todo.pop()
        if v in seen:
            continue
        seen.add(v)
        if v > num_pis:
            a, b = fanins[v - num_pis - 1]
            todo += [int(a) >> 1, int(b) >> 1]
    return seen


def priority_cuts(num_pis: int, fanins, need: set, k_l: int, C: int, pass_id: int,
                  repr_of: Dict[int, int]) -> Dict[int, List[Tuple[int, ...]]]:
    A = len(fanins)
    N = 1 + num_pis + A
    fanout = [0] * N
    level = [0] * N
    for j in range(A):
        a, b = int(fanins[j][0]) >> 1, int(fanins[j][1]) >> 1
        fanout[a] += 1
        fanout[b] += 1
        level[1 + num_pis + j] = 1 + max(level[a], level[b])

    def trivial(i):
        return () if i == 0 else (i,)

    P: Dict[int, List[Tuple[int, ...]]] = {}
    for i in range(1, num_pis + 1):
        if i in need:
            P[i] = [(i,)]
    if 0 in need:
        P[0] = [()]

    def table1(c):
        mf = Fraction(sum(fanout[x] for x in c), len(c))
        ml = Fraction(sum(level[x] for x in c), len(c))
        if pass_id == 0:
            return (-mf, len(c), ml, c)
        if pass_id == 1:
            return (ml, len(c), -mf, c)
        return (-ml, len(c), -mf, c)

    for j in range(A):
        n = 1 + num_pis + j
        if n not in need:
            continue
        a, b = int(fanins[j][0]) >> 1, int(fanins[j][1]) >> 1
        E = set()
        for u in P[a] + [trivial(a)]:
            for v in P[b] + [trivial(b)]:
                c = tuple(sorted(set(u) | set(v)))
                if 0 < len(c) <= k_l and c != (n,):
                    E.add(c)
        kept: List[Tuple[int, ...]] = []
        for c in sorted(E, key=lambda x: (len(x), x)):
            if not any(set(d) <= set(c) for d in kept):
                kept.append(c)
        r = repr_of.get(n)
        if r is not None and P.get(r):
            Pr = P[r]

            def sim(c):
                return sum(Fraction(len(set(c) & set(d)), len(set(c) | set(d))) for d in Pr)

            kept.sort(key=lambda c: (-sim(c),) + table1(c))
        else:
            kept.sort(key=table1)
        P[n] = kept[:C]
    return P


def common_cuts(num_pis: int, fanins, repr_ids: Sequence[int], member_ids: Sequence[int], k_l: int, C: int,
                pass_id: int, max_cuts: int) -> List[List[Tuple[int, ...]]]:
    need = _tfi(num_pis, fanins, list(repr_ids) + list(member_ids))
    repr_of = {int(m): int(r) for r, m in zip(repr_ids, member_ids)}
    P = priority_cuts(num_pis, fanins, need, k_l, C, pass_id, repr_of)
    out = []
    for r, m in zip(repr_ids, member_ids):
        cs = set()
        for u in P[int(r)]:
            for v in P[int(m)]:
                c = tuple(sorted(set(u) | set(v)))
                if 0 < len(c) <= k_l:
                    cs.add(c)
        out.append(sorted(cs, key=lambda x: (len(x), x))[:max_cuts])
    return out
