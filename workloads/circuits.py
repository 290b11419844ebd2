"""Seeded synthetic miters for BASELINE.json's five configs (SURVEY.md §8(d) "Synthetic inputs").

Input generation only: every function here builds graph structure from a seed. Nothing here
simulates, computes truth tables or supports, or compares functions (that is the method; it lives
in the CUDA path and, independently, in oracle/).

A miter (§II-B) shares the PIs of circuit A and circuit B; its candidate PO pairs are
(PO_A[i], PO_B[i]). We keep A and B structurally separate (two builders, concatenated) and list the
pairs as literal pairs instead of adding XOR gates, which the ABI accepts directly.
"""
from __future__ import annotations

import dataclasses
from typing import Callable, Dict, List, Optional, Sequence, Tuple

import numpy as np

from .aig import Aig, Builder

# ---------------------------------------------------------------------------------------------
# Miter container and concatenation
# ---------------------------------------------------------------------------------------------


@dataclasses.dataclass
class Miter:
    aig: Aig
    lit_a: np.ndarray  # uint32 [P]
    lit_b: np.ndarray  # uint32 [P]
    name: str = ""
    meta: dict = dataclasses.field(default_factory=dict)

    @property
    def num_pairs(self) -> int:
        return int(self.lit_a.size)


def _remap_lits(lits: np.ndarray, num_pis: int, pi_base: int, and_base: int) -> np.ndarray:
    """Remap literals of a local AIG (PIs 1..num_pis, ANDs after) into a global numbering where
    the local PI i maps to pi_base + i and the local AND j (id num_pis+1+j) to and_base + j."""
    lits = lits.astype(np.int64)
    ids = lits >> 1
    neg = lits & 1
    out = np.where(ids == 0, 0, np.where(ids <= num_pis, pi_base + ids, and_base + (ids - num_pis - 1)))
    return (2 * out + neg).astype(np.uint32)


def concat_miter(a: Aig, b: Aig, name: str = "") -> Miter:
    """Miter of A and B over the shared PIs, structurally hashed like an ABC miter: A's ANDs first,
    then B's ANDs re-created through the same hashing builder, so a B node identical to an A node
    (same fanin literals) is not duplicated. Pairs = (PO_A[i], PO_B[i]).
    meta: a_ands = #ANDs of A; b_ands = #ANDs created for B only (ids after A's)."""
    if a.num_pis != b.num_pis or a.pos.size != b.pos.size:
        raise ValueError("A and B must have the same PIs and PO count")
    I = a.num_pis
    bd = Builder(I, strash=True)
    for l0, l1 in a.fanins:
        bd.raw_and(int(l0), int(l1))
        bd._table[(min(int(l0), int(l1)), max(int(l0), int(l1)))] = 2 * (bd.next_id() - 1)
    a_ands = len(bd.ands)
    lit_map = np.zeros(1 + I + b.num_ands, dtype=np.int64)
    lit_map[1:1 + I] = 2 * np.arange(1, I + 1)
    for j, (l0, l1) in enumerate(b.fanins):
        x = int(lit_map[int(l0) >> 1]) ^ (int(l0) & 1)
        y = int(lit_map[int(l1) >> 1]) ^ (int(l1) & 1)
        lit_map[1 + I + j] = bd.AND(x, y)
    pb = np.array([int(lit_map[int(l) >> 1]) ^ (int(l) & 1) for l in b.pos], dtype=np.uint32)
    aig = bd.finish(list(a.pos) + list(pb))
    return Miter(aig, a.pos.astype(np.uint32).copy(), pb, name=name,
                 meta={"a_ands": a_ands, "b_ands": len(bd.ands) - a_ands, "b_lit_map": lit_map})


def b_image(miter_a_ands: int, num_pis: int, lit_in_b: int) -> int:
    """Global literal of a literal expressed in B's local numbering (helper for internal pairs)."""
    return int(_remap_lits(np.array([lit_in_b], dtype=np.uint32), num_pis, 0, 1 + num_pis + miter_a_ands)[0])


# ---------------------------------------------------------------------------------------------
# Adders (C1, C4)
# ---------------------------------------------------------------------------------------------

def ripple_adder(bd: Builder, a: Sequence[int], b: Sequence[int], cin: Optional[int] = None,
                 alt: bool = False) -> Tuple[List[int], int]:
    """Ripple-carry adder: s_i = a_i ^ b_i ^ c_i, c_{i+1} = MAJ(a_i, b_i, c_i)."""
    xor = bd.XOR_alt if alt else bd.XOR
    s: List[int] = []
    c = cin
    for ai, bi in zip(a, b):
        if c is None:  # half adder
            s.append(xor(ai, bi))
            c = bd.AND(ai, bi)
        else:
            p = xor(ai, bi)
            s.append(xor(p, c))
            c = bd.OR(bd.AND(ai, bi), bd.AND(p, c))
    return s, (c if c is not None else 0)


def kogge_stone_adder(bd: Builder, a: Sequence[int], b: Sequence[int]) -> Tuple[List[int], int]:
    """Kogge-Stone parallel-prefix adder: g = a&b, p = a^b; log2(n) prefix stages;
    s_0 = p_0, s_i = p_i ^ G_{i-1:0}, cout = G_{n-1:0}."""
    n = len(a)
    g = [bd.AND(x, y) for x, y in zip(a, b)]
    p = [bd.XOR(x, y) for x, y in zip(a, b)]
    G, P = list(g), list(p)
    d = 1
    while d < n:
        G2, P2 = list(G), list(P)
        for i in range(d, n):
            G2[i] = bd.OR(G[i], bd.AND(P[i], G[i - d]))
            P2[i] = bd.AND(P[i], P[i - d])
        G, P = G2, P2
        d *= 2
    s = [p[0]] + [bd.XOR(p[i], G[i - 1]) for i in range(1, n)]
    return s, G[n - 1]


def block_cla_adder(bd: Builder, a: Sequence[int], b: Sequence[int], cin: int, block: int = 4
                    ) -> Tuple[List[int], int]:
    """Block carry-lookahead adder: per block, group generate/propagate; carries ripple between
    blocks through the group signals; inside a block carries are flattened lookahead terms."""
    n = len(a)
    g = [bd.AND(x, y) for x, y in zip(a, b)]
    p = [bd.XOR_alt(x, y) for x, y in zip(a, b)]
    s: List[int] = []
    c = cin
    for lo in range(0, n, block):
        hi = min(n, lo + block)
        carry_in_bit = c  # carry into bit i, expressed from the block's carry-in c
        for i in range(lo, hi):
            s.append(bd.XOR_alt(p[i], carry_in_bit))
            # lookahead: c_{i+1} = g_i + p_i g_{i-1} + ... + p_i..p_lo c
            terms = [g[i]]
            pp = p[i]
            for j in range(i - 1, lo - 1, -1):
                terms.append(bd.AND(pp, g[j]))
                pp = bd.AND(pp, p[j])
            terms.append(bd.AND(pp, c))
            acc = terms[0]
            for t in terms[1:]:
                acc = bd.OR(acc, t)
            carry_in_bit = acc
        c = carry_in_bit
    return s, c


# ---------------------------------------------------------------------------------------------
# Multipliers (C2)
# ---------------------------------------------------------------------------------------------

def array_multiplier(bd: Builder, a: Sequence[int], b: Sequence[int]) -> List[int]:
    """Row-by-row array multiplier: acc += (a & b_i) << i with a ripple row adder per row."""
    n, m = len(a), len(b)
    acc = [0] * (n + m)
    for j in range(n):
        acc[j] = bd.AND(a[j], b[0])
    for i in range(1, m):
        row = [bd.AND(a[j], b[i]) for j in range(n)]
        s, c = ripple_adder(bd, acc[i:i + n], row, None)
        acc[i:i + n] = s
        acc[i + n] = c
    return acc


def wallace_multiplier(bd: Builder, a: Sequence[int], b: Sequence[int], bug: Optional[dict] = None
                       ) -> List[int]:
    """Wallace-tree multiplier: partial-product columns reduced by full/half adders (3:2 and 2:2
    counters) until height 2, then a Kogge-Stone final adder. Uses the alternative XOR/MAJ forms so
    the B side differs structurally from the array multiplier."""
    n, m = len(a), len(b)
    W = n + m
    cols: List[List[int]] = [[] for _ in range(W + 1)]
    for i in range(m):
        for j in range(n):
            cols[i + j].append(bd.AND(a[j], b[i]))
    while max(len(c) for c in cols) > 2:
        new: List[List[int]] = [[] for _ in range(W + 1)]
        for w in range(W):
            bits = cols[w]
            k = 0
            while len(bits) - k >= 3:
                x, y, z = bits[k:k + 3]
                k += 3
                t = bd.XOR_alt(x, y)
                new[w].append(bd.XOR_alt(t, z))
                if w + 1 <= W:
                    new[w + 1].append(bd.MAJ_alt(x, y, z))
            if len(bits) - k == 2:
                x, y = bits[k:k + 2]
                new[w].append(bd.XOR_alt(x, y))
                new[w + 1].append(bd.AND(x, y))
            elif len(bits) - k == 1:
                new[w].append(bits[k])
        cols = new
    r0 = [c[0] if len(c) > 0 else 0 for c in cols[:W]]
    r1 = [c[1] if len(c) > 1 else 0 for c in cols[:W]]
    s, _ = kogge_stone_adder(bd, r0, r1)
    return s


# ---------------------------------------------------------------------------------------------
# Random block logic and function-preserving rewrites (C3, C5)
# ---------------------------------------------------------------------------------------------

def random_block(bd: Builder, pis: Sequence[int], n_ands: int, rng: np.random.Generator,
                 window: int = 64, p_pi: float = 0.1) -> List[int]:
    """Append n_ands ANDs. Each fanin comes from the block's last `window` nodes with probability
    1-p_pi, otherwise from the block's PIs; complements are Bernoulli(0.5)."""
    nodes: List[int] = []
    used: List[bool] = []
    tries = 0
    while len(nodes) < n_ands:
        tries += 1
        if tries > 50 * n_ands + 1000:
            raise RuntimeError("random_block: cannot make progress")
        fan = []
        lo = max(0, len(nodes) - window)
        # a node about to leave the fanin window without a fanout is used now, so that almost
        # every node ends up in some PO cone (few dangling nodes, like a real netlist)
        forced = lo if (nodes and len(nodes) >= window and not used[lo]) else -1
        for t in range(2):
            if t == 0 and forced >= 0:
                idx = forced
                v = nodes[idx]
            elif nodes and rng.random() >= p_pi:
                idx = int(rng.integers(lo, len(nodes)))
                v = nodes[idx]
            else:
                idx = -1
                v = pis[int(rng.integers(0, len(pis)))]
            fan.append((v ^ int(rng.integers(0, 2)), idx))
        if (fan[0][0] >> 1) == (fan[1][0] >> 1):
            continue
        before = len(bd.ands)
        lit = bd.AND(fan[0][0], fan[1][0])
        if len(bd.ands) == before:  # folded or hashed: not a new node
            continue
        for _, idx in fan:
            if idx >= 0:
                used[idx] = True
        nodes.append(lit)
        used.append(False)
    random_block.last_unused = [nodes[i] for i in range(len(nodes)) if not used[i]]
    return nodes


def rewrite_copy(src: Aig, rng: np.random.Generator, p_rw: float = 0.3,
                 node_map_out: Optional[Dict[int, int]] = None) -> Aig:
    """A function-preserving restructured copy of `src` (SURVEY.md §8(d) "Invariant rewrites must
    change structure"): with probability p_rw per node, re-associate an AND tree
    (x·(p·q) -> p·(q·x)) or distribute over a complemented fanin (y·!(p·q) -> y·!p + y·!q);
    every other node is copied. Rewrites never add structural support.

    node_map_out, if given, receives {src AND id: literal of its image in the returned AIG}."""
    I = src.num_pis
    bd = Builder(I, strash=True)
    lit_map = np.zeros(1 + I + src.num_ands, dtype=np.int64)
    lit_map[1:1 + I] = 2 * np.arange(1, I + 1)

    def m(l: int) -> int:
        return int(lit_map[l >> 1]) ^ (l & 1)

    def fan_of(lit: int):
        v = lit >> 1
        if v <= I:
            return None
        return bd.ands[v - I - 1]

    for j in range(src.num_ands):
        x, y = m(int(src.fanins[j, 0])), m(int(src.fanins[j, 1]))
        r = rng.random()
        out = None
        if r < p_rw:
            if rng.random() < 0.5:
                x, y = y, x
            fx = fan_of(x)
            if fx is not None and (x & 1) == 0:
                p, q = fx
                if rng.random() < 0.5:
                    p, q = q, p
                out = bd.AND(p, bd.AND(q, y))
            elif fx is not None:
                p, q = fx
                out = bd.OR(bd.AND(y, p ^ 1), bd.AND(y, q ^ 1))
        if out is None:
            out = bd.AND(x, y)
        lit_map[1 + I + j] = out
        if node_map_out is not None:
            node_map_out[1 + I + j] = out
    pos = [m(int(l)) for l in src.pos]
    return bd.finish(pos)


def random_miter(num_pis: int, n_ands: int, n_pos: int, seed: int, window: int = 64,
                 p_pi: float = 0.1, p_rw: float = 0.3) -> Miter:
    """Random-block circuit A and its rewritten copy B over the same PIs."""
    rng = np.random.default_rng(seed)
    bd = Builder(num_pis, strash=True)
    pis = [bd.pi(i) for i in range(num_pis)]
    nodes = random_block(bd, pis, n_ands, rng, window=window, p_pi=p_pi)
    # POs: the dangling nodes first (so every node is in some PO cone), then seeded tail nodes
    dangling = list(random_block.last_unused)
    rest = [x for x in nodes[-max(n_pos * 3, 64):] if x not in set(dangling)]
    extra = max(0, n_pos - len(dangling))
    pick = rng.choice(len(rest), size=min(extra, len(rest)), replace=False) if extra else []
    chosen = sorted(set(dangling[:n_pos]) | {rest[int(i)] for i in pick})
    pos = [x ^ int(rng.integers(0, 2)) for x in chosen]
    a = bd.finish(pos)
    b = rewrite_copy(a, rng, p_rw=p_rw)
    return concat_miter(a, b, name=f"rand{num_pis}x{n_ands}s{seed}")


# ---------------------------------------------------------------------------------------------
# Bug injection (SURVEY.md §8(d) "Bug injection")
# ---------------------------------------------------------------------------------------------

def flip_fanin(miter: Miter, and_id: int, which: int) -> Miter:
    """Single-gate bug (i): flip the complement bit of fanin `which` of AND node `and_id`."""
    fan = miter.aig.fanins.copy()
    j = and_id - miter.aig.num_pis - 1
    if not 0 <= j < fan.shape[0]:
        raise IndexError(and_id)
    fan[j, which] ^= 1
    aig = Aig(miter.aig.num_pis, fan, miter.aig.pos.copy())
    return Miter(aig, miter.lit_a.copy(), miter.lit_b.copy(), name=miter.name + f"_bug{and_id}.{which}",
                 meta=dict(miter.meta, bug=(and_id, which)))


def b_side_ids(miter: Miter) -> Tuple[int, int]:
    """[lo, hi) AND-id range of circuit B inside a concat_miter miter."""
    I = miter.aig.num_pis
    lo = 1 + I + miter.meta["a_ands"]
    return lo, lo + miter.meta["b_ands"]


# ---------------------------------------------------------------------------------------------
# The five configs
# ---------------------------------------------------------------------------------------------

def c1_add8() -> Miter:
    """C1: 8-bit ripple-carry vs Kogge-Stone adder; PIs a = 1..8, b = 9..16; 9 PO pairs."""
    n = 8
    A = Builder(2 * n)
    a = [A.pi(i) for i in range(n)]
    b = [A.pi(n + i) for i in range(n)]
    s, c = ripple_adder(A, a, b)
    ga = A.finish(s + [c])
    B = Builder(2 * n)
    s, c = kogge_stone_adder(B, [B.pi(i) for i in range(n)], [B.pi(n + i) for i in range(n)])
    gb = B.finish(s + [c])
    return concat_miter(ga, gb, name="c1_add8")


def c2_mul12(n: int = 12) -> Miter:
    """C2: n x n array vs Wallace-tree multiplier; PIs a = 1..n, b = n+1..2n; 2n PO pairs."""
    A = Builder(2 * n)
    ga = A.finish(array_multiplier(A, [A.pi(i) for i in range(n)], [A.pi(n + i) for i in range(n)]))
    B = Builder(2 * n)
    gb = B.finish(wallace_multiplier(B, [B.pi(i) for i in range(n)], [B.pi(n + i) for i in range(n)]))
    return concat_miter(ga, gb, name=f"c2_mul{n}")


def c2_mul12_bug(seed: int = 1, n: int = 12) -> Miter:
    """C2-bug: flip one fanin complement of a seeded AND inside B's (Wallace) reduction logic."""
    m = c2_mul12(n)
    lo, hi = b_side_ids(m)
    rng = np.random.default_rng(seed)
    # reduction tree = the middle of B's id range (after the partial products, before the final adder)
    npp = n * n
    tree_lo = lo + npp
    tree_hi = max(tree_lo + 1, hi - 6 * 2 * n)
    node = int(rng.integers(tree_lo, tree_hi))
    bug = flip_fanin(m, node, int(rng.integers(0, 2)))
    bug.name = f"c2_mul{n}_bug{seed}"
    return bug


def c4_dp(n: int = 64, bug: Optional[int] = None, block: int = 4) -> Miter:
    """C4: n-bit datapath: s = a + b + cin (n+1 POs), lt = (a < b), y = lt ? b : a (n POs).
    A: ripple-carry adder, ripple comparator, 2:1 mux. B: block-CLA adder, lt = NOT carry-out of
    a + ~b + 1, mux as a ^ (lt & (a ^ b)). PIs a = 1..n, b = n+1..2n, cin = 2n+1.
    bug=seed flips one complement inside block 5's group logic of B's adder (or the middle block
    for small n)."""
    I = 2 * n + 1
    A = Builder(I)
    a = [A.pi(i) for i in range(n)]
    b = [A.pi(n + i) for i in range(n)]
    s, c = ripple_adder(A, a, b, A.pi(2 * n))
    # ripple comparator from LSB: lt_{i+1} = (!a_i & b_i) | (!(a_i ^ b_i) & lt_i)
    lt = 0
    for i in range(n):
        eq = A.XOR(a[i], b[i]) ^ 1
        lt = A.OR(A.AND(a[i] ^ 1, b[i]), A.AND(eq, lt))
    y = [A.MUX(lt, b[i], a[i]) for i in range(n)]
    ga = A.finish(s + [c, lt] + y)

    B = Builder(I)
    a = [B.pi(i) for i in range(n)]
    b = [B.pi(n + i) for i in range(n)]
    s, c = block_cla_adder(B, a, b, B.pi(2 * n), block=block)
    # a - b = a + ~b + 1; carry-out = 1 iff a >= b
    _, cb = ripple_adder(B, a, [x ^ 1 for x in b], 1, alt=True)
    ltb = cb ^ 1
    y = [B.XOR(a[i], B.AND(ltb, B.XOR(a[i], b[i]))) for i in range(n)]
    gb = B.finish(s + [c, ltb] + y)
    m = concat_miter(ga, gb, name=f"c4_dp{n}")
    if bug is not None:
        lo, hi = b_side_ids(m)
        rng = np.random.default_rng(bug)
        # B's adder is built first: block 5 (bits 20..23 for block=4) sits roughly at 5/(n/block)
        nb = max(1, n // block)
        blk = min(5, nb - 1)
        adder_ands = None
        span = hi - lo
        # adder occupies the first part of B; pick inside block `blk` of it proportionally
        frac_lo = blk / nb
        frac_hi = (blk + 1) / nb
        adder_span = int(span * 0.5)
        node = int(rng.integers(lo + int(adder_span * frac_lo), lo + max(int(adder_span * frac_hi), int(adder_span * frac_lo) + 1)))
        m = flip_fanin(m, node, int(rng.integers(0, 2)))
        m.name = f"c4_dp{n}_bug{bug}"
    return m


def tiny_random(num_pis: int, n_ands: int, n_pairs: int, seed: int) -> Miter:
    """Small random AIG with random node-literal pairs, for brute-force fuzzing (<= 12 PIs)."""
    rng = np.random.default_rng(seed)
    bd = Builder(num_pis, strash=False)
    pis = [bd.pi(i) for i in range(num_pis)]
    nodes: List[int] = []
    for _ in range(n_ands):
        pool = pis + nodes
        x = pool[int(rng.integers(0, len(pool)))] ^ int(rng.integers(0, 2))
        y = pool[int(rng.integers(0, len(pool)))] ^ int(rng.integers(0, 2))
        nodes.append(bd.raw_and(x, y))
    allv = [0] + pis + nodes
    la = [allv[int(rng.integers(0, len(allv)))] ^ int(rng.integers(0, 2)) for _ in range(n_pairs)]
    lb = [allv[int(rng.integers(0, len(allv)))] ^ int(rng.integers(0, 2)) for _ in range(n_pairs)]
    aig = bd.finish(nodes[-4:] if nodes else [])
    return Miter(aig, np.array(la, dtype=np.uint32), np.array(lb, dtype=np.uint32), name=f"tiny{seed}")


def replicate(bases: Sequence[Miter], types: Sequence[int], name: str = "") -> Miter:
    """Disjoint copies (ABC `double`-style): copy c is bases[types[c]] with its own
    PIs (block of num_pis ids) and its own ANDs. All bases must have the same PI count."""
    I0 = bases[0].aig.num_pis
    for bm in bases:
        if bm.aig.num_pis != I0:
            raise ValueError("all base types must have the same PI count")
    C = len(types)
    I = I0 * C
    total_ands = sum(bases[t].aig.num_ands for t in types)
    fan = np.empty((total_ands, 2), dtype=np.uint32)
    la, lb, pos = [], [], []
    off = 0
    copy_and_base = []
    for c, t in enumerate(types):
        bm = bases[t]
        A = bm.aig.num_ands
        and_base = 1 + I + off
        fan[off:off + A] = _remap_lits(bm.aig.fanins, I0, c * I0, and_base)
        la.append(_remap_lits(bm.lit_a, I0, c * I0, and_base))
        lb.append(_remap_lits(bm.lit_b, I0, c * I0, and_base))
        pos.append(_remap_lits(bm.aig.pos, I0, c * I0, and_base))
        copy_and_base.append(and_base)
        off += A
    aig = Aig(I, fan, np.concatenate(pos).astype(np.uint32))
    aig.validate()
    return Miter(aig, np.concatenate(la).astype(np.uint32), np.concatenate(lb).astype(np.uint32), name=name,
                 meta={"types": list(types), "copy_and_base": copy_and_base,
                       "pairs_per_copy": [int(bases[t].num_pairs) for t in types]})


def c5_big(copies: int = 256, n_random: int = 176, seed: int = 5, n_bugs: int = 8,
           rand_ands: int = 4450, rand_pis: int = 24, rand_pos: int = 25, window: int = 80,
           mul_n: int = 12) -> Miter:
    """C5: ~2M-node miter of disjoint copies shaped like sin_10xd per copy (24 PIs, ~25 POs, ~10.4k
    miter ANDs, ~225 levels) plus mul12 miter copies. `n_bugs` copies get a
    single-gate bug: one fanin complement of the B-side AND driving a seeded PO is flipped."""
    rng = np.random.default_rng(seed)
    bases = [random_miter(rand_pis, rand_ands, rand_pos, seed=1000 * seed + t, window=window) for t in range(3)]
    bases.append(c2_mul12(mul_n))
    n_mul = copies - n_random
    types = [t % 3 for t in range(n_random)] + [3] * n_mul
    types = [int(x) for x in rng.permutation(types)]
    bug_copies = sorted(int(x) for x in rng.choice(copies, size=min(n_bugs, copies), replace=False))
    all_bases = list(bases)
    for c in bug_copies:
        bm = bases[types[c]]
        lo, hi = b_side_ids(bm)
        cand = [p for p in range(bm.num_pairs) if lo <= (int(bm.lit_b[p]) >> 1) < hi]
        if not cand:
            continue
        p = cand[int(rng.integers(0, len(cand)))]
        drv = int(bm.lit_b[p]) >> 1
        bugged = flip_fanin(bm, drv, int(rng.integers(0, 2)))
        all_bases.append(bugged)
        types[c] = len(all_bases) - 1
    m = replicate(all_bases, types, name=f"c5_big{copies}")
    m.meta["bug_copies"] = bug_copies
    m.meta["base_types"] = len(bases)
    return m


def c3_rand(seed: int = 3, sample_seed: int = 7, n_blocks: int = 200, block_ands: int = 500, num_pis: int = 1024,
            n_internal: int = 5000, n_near: int = 64, k_dist=((150, 12, 20), (40, 21, 26), (8, 27, 31), (2, 32, 32)),
            window: int = 64, p_rw: float = 0.3) -> Miter:
    """C3: random block AIG A (blocks of ~block_ands ANDs, block b reads a contiguous
    window of k_b PIs out of num_pis; fanins from the block's last `window` nodes w.p. 0.9 else its
    PIs; up to 8 dangling nodes per block become POs) vs its rewritten copy B. Pairs: every PO
    pair, n_internal sampled (A node, B image) pairs and n_near near-miss pairs (A node vs its B
    image with one fanin complemented: appended nodes, mostly NEQ)."""
    rng = np.random.default_rng(seed)
    ks = []
    for cnt, lo, hi in k_dist:
        ks += [int(x) for x in rng.integers(lo, hi + 1, size=cnt)]
    ks = [int(x) for x in rng.permutation(ks)][:n_blocks]
    bd = Builder(num_pis, strash=True)
    pos: List[int] = []
    for kb in ks:
        start = int(rng.integers(0, num_pis - kb + 1))
        pis = [bd.pi(start + i) for i in range(kb)]
        random_block(bd, pis, block_ands, rng, window=window, p_pi=0.1)
        dang = list(random_block.last_unused)[-8:]
        pos += [x ^ int(rng.integers(0, 2)) for x in dang]
    a = bd.finish(pos)
    img: Dict[int, int] = {}
    b = rewrite_copy(a, rng, p_rw=p_rw, node_map_out=img)
    m = concat_miter(a, b, name=f"c3_rand{n_blocks}x{block_ands}")
    bmap = m.meta["b_lit_map"]
    I = num_pis

    def b_lit(local_lit: int) -> int:
        return int(bmap[local_lit >> 1]) ^ (local_lit & 1)

    srng = np.random.default_rng(sample_seed)
    a_ids = np.arange(1 + I, 1 + I + a.num_ands)
    la = [int(x) for x in m.lit_a]
    lb = [int(x) for x in m.lit_b]
    cand = [int(x) for x in srng.permutation(a_ids)]
    internal = 0
    for nid in cand:
        if internal >= n_internal:
            break
        il = b_lit(img[nid])
        if il == 2 * nid:
            continue  # hashed onto the A node itself: trivially equal
        la.append(2 * nid)
        lb.append(il)
        internal += 1
    fan = [tuple(int(v) for v in r) for r in m.aig.fanins]
    near = 0
    for nid in cand[::-1]:
        if near >= n_near:
            break
        il = b_lit(img[nid])
        v = il >> 1
        if v <= I or il == 2 * nid:
            continue
        f0, f1 = fan[v - I - 1]
        fan.append((f0 ^ 1, f1))
        new_id = 1 + I + len(fan) - 1
        la.append(2 * nid)
        lb.append(2 * new_id ^ (il & 1))
        near += 1
    aig = Aig(I, np.asarray(fan, dtype=np.uint32).reshape(-1, 2), m.aig.pos.copy())
    aig.validate()
    meta = dict(m.meta)
    meta.pop("b_lit_map", None)
    meta.update({"k_blocks": ks, "po_pairs": len(m.lit_a), "internal_pairs": internal, "near_pairs": near})
    return Miter(aig, np.asarray(la, dtype=np.uint32), np.asarray(lb, dtype=np.uint32), name=m.name, meta=meta)
