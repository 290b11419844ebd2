"""Pins of the miter-reduction oracle (oracle/reduce.py, PAPER.md:61/:185/:187) against things other
than itself: hand-worked examples, functional equivalence of every old node with its image checked
by the independent brute-force evaluator (oracle/brute.py), the strash invariants of the result,
idempotence and identity on a structurally hashed AIG. CPU only."""
import numpy as np
import pytest

from oracle import brute
from oracle.reduce import reduce_miter
from workloads import c1_add8, tiny_random


def vectors(num_pis, fanins):
    """Value of every node id on every one of the 2^num_pis assignments (brute.eval_all)."""
    fan = [(int(a), int(b)) for a, b in fanins]
    rows = [brute.eval_all(num_pis, fan, {1 + t: (u >> t) & 1 for t in range(num_pis)})
            for u in range(1 << num_pis)]
    return np.array(rows, dtype=np.uint8).T  # [node id, assignment]


def lit_vec(vec, lit):
    return vec[lit >> 1] ^ (lit & 1)


def check_structure(num_pis, out):
    """AIGER-binary order, no trivial AND, no duplicate fanin pair, fanins sorted."""
    seen = set()
    for j, (a, b) in enumerate(out):
        nid = 1 + num_pis + j
        assert a < b and (b >> 1) < nid
        assert a > 1 and a != b and a != b ^ 1
        assert (a, b) not in seen
        seen.add((a, b))


def test_hand_duplicates_and_trivial():
    # x=1, y=2; n3 = x&y, n4 = y&x (duplicate), n5 = n3&n4 (= n3 after hashing), n6 = x & !x
    fan = [(2, 4), (4, 2), (6, 8), (2, 3)]
    out, image, lits = reduce_miter(2, fan, {}, [10, 11, 12])
    assert out == [(2, 4)]
    assert image == [0, 2, 4, 6, 6, 6, 0]
    assert lits == [6, 7, 0]


def test_hand_redirect_member_to_representative():
    # n3 = x&y, n4 = !x&!y, n5 = n3 & !n4 (= n3); proving (n3, n5) equal merges n5 into n3
    fan = [(2, 4), (3, 5), (6, 9)]
    out, image, _ = reduce_miter(2, fan, {5: 6})
    assert out == [(2, 4), (3, 5)]
    assert image == [0, 2, 4, 6, 8, 6]
    # a fanout of the member is redirected: n6 = n5 & y  ->  (x&y)&y, built on n3
    fan2 = fan + [(10, 4)]
    out2, image2, _ = reduce_miter(2, fan2, {5: 6})
    assert out2 == [(2, 4), (3, 5), (4, 6)] and image2[6] == 10
    # a member merged into a complemented representative and into the constant
    out3, image3, _ = reduce_miter(2, fan, {4: 7, 5: 0})
    assert out3 == [(2, 4)] and image3[4] == 7 and image3[5] == 0


def test_representative_must_be_lower():
    with pytest.raises(ValueError):
        reduce_miter(2, [(2, 4), (3, 5)], {3: 8})


def _functional_subst(num_pis, fanins, vec):
    """Every AND merged into the minimum id with an identical or complementary vector (exact
    classes from brute-force vectors)."""
    first = {}
    subst = {}
    for nid in range(vec.shape[0]):
        key, inv = vec[nid].tobytes(), (1 - vec[nid]).tobytes()
        if key in first:
            if nid > num_pis:
                subst[nid] = 2 * first[key]
        elif inv in first:
            if nid > num_pis:
                subst[nid] = 2 * first[inv] + 1
        else:
            first[key] = nid
    return subst


@pytest.mark.parametrize("seed", range(12))
def test_images_are_functionally_equal(seed):
    m = tiny_random(num_pis=3 + seed % 6, n_ands=40 + 7 * seed, n_pairs=1, seed=200 + seed)
    I, fan = m.aig.num_pis, [tuple(map(int, r)) for r in m.aig.fanins]
    vec = vectors(I, fan)
    rng = np.random.default_rng(seed)
    for subst in ({}, _functional_subst(I, fan, vec)):
        # also a random half of the functional merges (any subset is a valid reduction)
        for sub in (subst, {k: v for k, v in subst.items() if rng.random() < 0.5}):
            out, image, _ = reduce_miter(I, fan, sub)
            check_structure(I, out)
            nvec = vectors(I, out)
            for nid in range(1 + I + len(fan)):
                assert np.array_equal(vec[nid], lit_vec(nvec, image[nid])), (seed, nid)
            # idempotence: reducing the result again with no merges changes nothing
            out2, image2, _ = reduce_miter(I, out, {})
            assert out2 == out and image2 == [0] + [2 * i for i in range(1, 1 + I + len(out))]
    # full functional merge: surviving ANDs have pairwise different functions up to complement
    out, _, _ = reduce_miter(I, fan, _functional_subst(I, fan, vec))
    nvec = vectors(I, out)
    keys = set()
    for nid in range(1 + I, 1 + I + len(out)):
        k = min(nvec[nid].tobytes(), (1 - nvec[nid]).tobytes())
        assert k not in keys
        keys.add(k)


def test_identity_on_hashed_miter():
    m = c1_add8()  # built with strash: reduction without merges is the identity
    I, fan = m.aig.num_pis, [tuple(map(int, r)) for r in m.aig.fanins]
    out, image, lits = reduce_miter(I, fan, {}, list(m.lit_a))
    assert out == [tuple(sorted(f)) for f in fan]
    assert lits == [int(x) for x in m.lit_a]
