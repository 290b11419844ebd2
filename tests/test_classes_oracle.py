"""Pins of the equivalence-class oracle (oracle/classes.py, PAPER.md:41/:61/:183/:187): the
published splitmix64 output sequence, exact functional classes of the independent brute-force
evaluator when the patterns are the whole input cube, hand cases. CPU only."""
import numpy as np
import pytest

import oracle
from oracle import brute
from oracle.classes import classes, pattern_words, splitmix64
from workloads import Builder, tiny_random


def test_splitmix64_published_sequence():
    # splitmix64 with state 0 (Vigna's reference splitmix64.c): the first four outputs
    g = 0x9E3779B97F4A7C15
    want = [0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4, 0x06C45D188009454F, 0xF88BB8A8724C81EC]
    assert [splitmix64((k * g) % (1 << 64)) for k in range(4)] == want


def cube_words(num_pis):
    """Caller patterns covering all 2^num_pis assignments: pattern u = assignment u (PI i+1 = bit i)."""
    P = 1 << num_pis
    W = (P + 31) // 32
    words = np.zeros((num_pis, W), dtype=np.uint32)
    for u in range(P):
        for i in range(num_pis):
            if (u >> i) & 1:
                words[i, u // 32] |= np.uint32(1 << (u % 32))
    return words


def brute_classes(num_pis, fanins):
    """Exact classes of functions up to complement by full enumeration (brute.eval_all)."""
    fan = [(int(a), int(b)) for a, b in fanins]
    P = 1 << num_pis
    tabs = [brute.eval_all(num_pis, fan, {1 + t: (u >> t) & 1 for t in range(num_pis)}) for u in range(P)]
    N = 1 + num_pis + len(fan)
    first, out = {}, []
    for n in range(N):
        vec = tuple(tabs[u][n] for u in range(P))
        comp = tuple(1 - x for x in vec)
        if vec in first:
            if n > num_pis:
                out.append((first[vec][0], n, first[vec][1]))
        elif comp in first:
            if n > num_pis:
                out.append((first[comp][0], n, 1 ^ first[comp][1]))
        else:
            first[vec] = (n, 0)
    return out


@pytest.mark.parametrize("seed", range(10))
def test_full_cube_patterns_give_functional_classes(seed):
    m = tiny_random(num_pis=2 + seed % 7, n_ands=30 + 9 * seed, n_pairs=1, seed=500 + seed)
    orc = oracle.Oracle.from_aig(m.aig)
    got = classes(orc, num_words=0, seed=0, pi_words=cube_words(m.aig.num_pis))
    assert got == brute_classes(m.aig.num_pis, m.aig.fanins)


def test_random_patterns_refine_nothing_that_is_equal():
    # functional equivalences survive any pattern set: every exact class member is paired with
    # the same representative under random patterns too (random patterns may add false members)
    for seed in range(6):
        m = tiny_random(num_pis=6, n_ands=80, n_pairs=1, seed=600 + seed)
        orc = oracle.Oracle.from_aig(m.aig)
        got = {(r, n, f) for r, n, f in classes(orc, num_words=2, seed=seed)}
        want = brute_classes(m.aig.num_pis, m.aig.fanins)
        mem = {n: (r, f) for r, n, f in got}
        for r, n, f in want:
            assert mem.get(n) is not None
            # n's random-pattern representative is its exact representative or an id below it
            assert mem[n][0] <= r


def test_hand_cases():
    bd = Builder(2, strash=False)
    x, y = bd.pi(0), bd.pi(1)
    a = bd.raw_and(x, y)          # id 3
    b = bd.raw_and(y, x)          # id 4 = n3
    c = bd.raw_and(x, x ^ 1)      # id 5 = const 0
    d = bd.raw_and(x ^ 1, y ^ 1)  # id 6 = !(x | y)
    e = bd.raw_and(d ^ 1, a ^ 1)  # id 7 = (x|y) & !(x&y) = x ^ y
    f = bd.raw_and(a ^ 1, d ^ 1)  # id 8 = same as n7
    aig = bd.finish([e, f])
    orc = oracle.Oracle.from_aig(aig)
    got = classes(orc, num_words=0, seed=0, pi_words=cube_words(2))
    assert got == [(3, 4, 0), (0, 5, 0), (7, 8, 0)]
    # random words: the class structure is the same for this tiny AIG (4 assignments all appear)
    assert classes(orc, num_words=1, seed=9) == got


def test_pattern_words_layout():
    w = pattern_words(3, 2, 11, np.array([[1], [2], [3]], dtype=np.uint32))
    assert [len(r) for r in w] == [3, 3, 3]
    assert w[1][0] == splitmix64(11 ^ (2 << 32) ^ 0) & 0xFFFFFFFF
    assert [r[2] for r in w] == [1, 2, 3]
