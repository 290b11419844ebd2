"""brute — TEST INFRASTRUCTURE ONLY. An independent pure-Python brute-force enumerator used to pin the
C oracle (task rule ③: "brute force on tiny inputs"). It shares no code with oracle.c or with the
product: its own TFI walk, its own evaluator over *all* 2^I full PI assignments (I <= 12), and a
different route to the canonical CEX (collect every mismatching full assignment, keep those whose
non-support PIs are 0, project onto the support with pext, take the minimum — SURVEY.md §8(c) Q8).
"""
from __future__ import annotations

from typing import Dict, List, Sequence, Tuple

UND, EQ, NEQ = 0, 1, 2


def tfi(num_pis: int, fanins: Sequence[Tuple[int, int]], roots: Sequence[int], stop=frozenset()) -> set:
    seen = set()
    todo = list(roots)
    while todo:
        v = todo.pop()
        if v in seen:
            continue
        seen.add(v)
        if v in stop or v <= num_pis:
            continue
        a, b = fanins[v - num_pis - 1]
        todo += [a >> 1, b >> 1]
    return seen


def eval_all(num_pis: int, fanins: Sequence[Tuple[int, int]], assign: Dict[int, int]) -> List[int]:
    """Values of every node id under a PI assignment {pi_id: bit}; const0 = 0."""
    val = [0] * (1 + num_pis + len(fanins))
    for pid, b in assign.items():
        val[pid] = b
    for j, (a, b) in enumerate(fanins):
        va = val[a >> 1] ^ (a & 1)
        vb = val[b >> 1] ^ (b & 1)
        val[1 + num_pis + j] = va & vb
    return val


def lit_val(val: List[int], lit: int) -> int:
    return val[lit >> 1] ^ (lit & 1)


def check_pairs(num_pis: int, fanins, pairs: Sequence[Tuple[int, int]], k_max: int = 32):
    """Returns [(k, verdict, cex_or_None)] per pair, by full enumeration of all 2^num_pis inputs."""
    assert num_pis <= 12, "brute force is for tiny circuits only"
    fan = [(int(a), int(b)) for a, b in fanins]
    tables = []
    for u in range(1 << num_pis):
        tables.append(eval_all(num_pis, fan, {1 + t: (u >> t) & 1 for t in range(num_pis)}))
    out = []
    for la, lb in pairs:
        S = sorted(v for v in tfi(num_pis, fan, [la >> 1, lb >> 1]) if 1 <= v <= num_pis)
        k = len(S)
        if k > k_max:
            out.append((k, UND, None))
            continue
        mism = [u for u in range(1 << num_pis) if lit_val(tables[u], la) != lit_val(tables[u], lb)]
        # structural support contains every functional dependency: flipping a non-support PI
        # never changes whether an assignment mismatches (sanity property of the definition)
        nonsup_mask = sum(1 << (p - 1) for p in range(1, num_pis + 1) if p not in S)
        own = []
        for u in mism:
            if u & nonsup_mask:
                continue
            own.append(sum(((u >> (S[j] - 1)) & 1) << j for j in range(k)))  # pext onto S
        if own:
            out.append((k, NEQ, min(own)))
        else:
            assert not mism, "mismatch depends on a PI outside the structural support"
            out.append((k, EQ, None))
    return out


def check_local(num_pis: int, fanins, la: int, lb: int, leaves: Sequence[int]):
    """EQ if the local functions over `leaves` agree on every leaf assignment, UND otherwise,
    'BADCUT' if a root's cone reaches a PI that is not a leaf."""
    fan = [(int(a), int(b)) for a, b in fanins]
    L = sorted(set(int(x) for x in leaves))
    cone = tfi(num_pis, fan, [la >> 1, lb >> 1], stop=frozenset(L))
    if any(1 <= v <= num_pis and v not in L for v in cone):
        return "BADCUT"
    for i in range(1 << len(L)):
        val = {}
        for j, x in enumerate(L):
            val[x] = (i >> j) & 1

        def ev(v):
            if v == 0:
                return 0
            if v in val:
                return val[v]
            a, b = fan[v - num_pis - 1]
            r = (ev(a >> 1) ^ (a & 1)) & (ev(b >> 1) ^ (b & 1))
            val[v] = r
            return r

        if (ev(la >> 1) ^ (la & 1)) != (ev(lb >> 1) ^ (lb & 1)):
            return UND
    return EQ
