"""GPU parity: the CUDA path (through the C-ABI) against the CPU oracle, element by element on the
same seeded inputs. Integer/bitwise path => bit-exact: verdicts, k, canonical CEX indices and CEX
vectors (zero tolerance)."""
import json
import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import oracle  # noqa: E402
from oracle import Oracle  # noqa: E402
from paper_conf_dac_liuy25_b200 import capi  # noqa: E402
from workloads import Builder, c1_add8, c2_mul12, c2_mul12_bug, c5_big, circuits, tiny_random  # noqa: E402

GOLD = os.path.join(os.path.dirname(__file__), "golden")
NO = oracle.NO_CEX


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def gpu_ctx(aig, **kw):
    return capi.Context.from_aig(aig, **kw)


def assert_same(gv, gc, gk, ov, oc, ok, tag=""):
    assert list(map(int, gk)) == list(map(int, ok)), f"{tag} k differs"
    assert list(map(int, gv)) == list(map(int, ov)), f"{tag} verdicts differ"
    gc = [int(c) if int(v) == oracle.NOT_EQUIVALENT else NO for v, c in zip(gv, gc)]
    oc = [int(c) if int(v) == oracle.NOT_EQUIVALENT else NO for v, c in zip(ov, oc)]
    assert gc == oc, f"{tag} CEX indices differ"


def check_vs_oracle(m, k_max=32, **kw):
    ctx = gpu_ctx(m.aig, k_max=k_max, **kw)
    gv, gc, gk = ctx.sim_exhaustive(m.lit_a, m.lit_b)
    orc = Oracle.from_aig(m.aig)
    ov, oc, ok, _ = orc.check_pairs(m.lit_a, m.lit_b, k_max=k_max)
    assert_same(gv, gc, gk, ov, oc, ok, m.name)
    for p in np.nonzero(gv == capi.CEC_NOT_EQUIVALENT)[0][:64]:
        vec = ctx.get_cex(int(p))
        assert np.array_equal(vec, orc.cex_vector(int(m.lit_a[p]), int(m.lit_b[p]), int(oc[p])))
        assert orc.eval_lit(int(m.lit_a[p]), vec) != orc.eval_lit(int(m.lit_b[p]), vec)
    return ctx, gv, gc, gk


def test_paper_examples_on_gpu():
    bd = Builder(3, strash=False)
    x, y, z = bd.pi(0), bd.pi(1), bd.pi(2)
    n4 = bd.raw_and(x, y ^ 1)
    n5 = bd.raw_and(n4, z)
    f = bd.raw_and(n4 ^ 1, n5 ^ 1) ^ 1
    s4 = bd.raw_and(x ^ 1, y ^ 1)  # SDC example: n1 = !s4
    s5 = bd.raw_and(y, z)
    s6 = bd.raw_and(s4 ^ 1, s5)
    aig = bd.finish([f])
    ctx = gpu_ctx(aig)
    v, c, k = ctx.sim_exhaustive([f, f, 0, s6, f], [n4, x, 1, s5, f ^ 1])
    assert list(v) == [capi.CEC_EQUIVALENT, capi.CEC_NOT_EQUIVALENT, capi.CEC_NOT_EQUIVALENT,
                       capi.CEC_EQUIVALENT, capi.CEC_NOT_EQUIVALENT]
    assert int(c[1]) == 3 and int(c[2]) == 0 and list(k[:3]) == [3, 3, 0]
    lv = ctx.check_local_cuts([s6, s6], [s5, s5], [0, 2, 5], [s4 >> 1, s5 >> 1, 1, 2, 3])
    assert list(lv) == [capi.CEC_UNDECIDED, capi.CEC_EQUIVALENT]  # PAPER.md:35/:130 SDC; cut = support


ENGINES = [capi.CEC_ENGINE_INTERP, capi.CEC_ENGINE_JIT, capi.CEC_ENGINE_SIMT]
SHARD_ENGINES = [capi.CEC_ENGINE_INTERP, capi.CEC_ENGINE_JIT]


@pytest.mark.parametrize("seed", range(60))
def test_fuzz_tiny_random(seed):
    rng = np.random.default_rng(seed)
    I = int(rng.integers(1, 13))
    m = tiny_random(I, int(rng.integers(1, 120)), 24, 7000 + seed)
    kmax = int(rng.integers(0, 13))
    merge = int(rng.integers(0, 3))
    check_vs_oracle(m, k_max=kmax, merge=merge, engine=ENGINES[seed % 3])


@pytest.mark.parametrize("engine", ENGINES)
def test_c1_add8(engine):
    check_vs_oracle(c1_add8(), engine=engine)


@pytest.mark.parametrize("engine", ENGINES)
@pytest.mark.parametrize("n", [6, 8, 10])
def test_small_multipliers_and_bugs(n, engine):
    check_vs_oracle(circuits.c2_mul12(n), engine=engine)
    check_vs_oracle(circuits.c2_mul12_bug(seed=1, n=n), engine=engine)
    check_vs_oracle(circuits.c2_mul12_bug(seed=3, n=n), merge=capi.CEC_MERGE_OFF, engine=engine)


def test_invariance_merge_kmax_engine():
    m = c5_big(copies=6, n_random=4, n_bugs=3, rand_pis=14, rand_ands=700, mul_n=7)
    ref = None
    for merge, k_max, engine in [(m_, k_, e_) for m_ in (capi.CEC_MERGE_OFF, capi.CEC_MERGE_PAPER, capi.CEC_MERGE_COST)
                                 for k_ in (32, 40) for e_ in ENGINES]:
        if True:
            ctx = gpu_ctx(m.aig, merge=merge, k_max=k_max, k_s=28 if merge else 0, engine=engine)
            got = ctx.sim_exhaustive(m.lit_a, m.lit_b)
            if ref is None:
                ref = got
                orc = Oracle.from_aig(m.aig)
                ov, oc, ok, _ = orc.check_pairs(m.lit_a, m.lit_b, k_max=32)
                assert_same(*got, ov, oc, ok, "c5-mini")
            else:
                for a, b in zip(ref, got):
                    assert np.array_equal(a, b)


@pytest.mark.parametrize("engine", ENGINES)
def test_c5_reduced_vs_oracle(engine):
    m = c5_big(copies=16, n_random=10, n_bugs=4, rand_pis=16, rand_ands=1500, mul_n=8)
    check_vs_oracle(m, engine=engine)


def _golden(name):
    path = os.path.join(GOLD, name + ".json")
    if not os.path.exists(path):
        pytest.skip(f"{path} missing (run scripts/make_golden.py)")
    return json.load(open(path))


@pytest.mark.parametrize("engine", ENGINES)
@pytest.mark.parametrize("name,fn", [("c2_mul12", lambda: c2_mul12()), ("c2_mul12_bug1", lambda: c2_mul12_bug(seed=1))])
def test_c2_full_vs_stored_oracle(name, fn, engine):
    g = _golden(name)
    m = fn()
    assert [int(x) for x in m.lit_a] == g["lit_a"] and [int(x) for x in m.lit_b] == g["lit_b"]
    assert int(m.aig.num_ands) == g["num_ands"]
    ctx = gpu_ctx(m.aig, engine=engine)
    gv, gc, gk = ctx.sim_exhaustive(m.lit_a, m.lit_b)
    assert_same(gv, gc, gk, g["verdict"], g["cex"], g["k"], name)
    orc = Oracle.from_aig(m.aig)
    for p in np.nonzero(gv == capi.CEC_NOT_EQUIVALENT)[0]:
        vec = ctx.get_cex(int(p))
        n = 12
        a = sum(int(vec[i]) << i for i in range(n))
        b = sum(int(vec[n + i]) << i for i in range(n))
        assert orc.eval_lit(int(m.lit_a[p]), vec) == ((a * b) >> int(p)) & 1  # closed form side
        assert orc.eval_lit(int(m.lit_b[p]), vec) != ((a * b) >> int(p)) & 1


def test_c5_full_size_sampled():
    """Full BASELINE C5 size in the bench's launch configuration: copy invariance for every copy and
    oracle confirmation of sampled outputs (every NEQ CEX re-derived as the first mismatch by the
    oracle scanning [0, cex]; EQ pairs of bug copies checked on a sampled pattern range)."""
    m = c5_big()
    ctx = gpu_ctx(m.aig)
    gv, gc, gk = ctx.sim_exhaustive(m.lit_a, m.lit_b)
    types = m.meta["types"]
    ppc = m.meta["pairs_per_copy"]
    off = np.concatenate([[0], np.cumsum(ppc)])
    by_type = {}
    for c, t in enumerate(types):
        sl = slice(off[c], off[c + 1])
        sig = (tuple(gv[sl]), tuple(gc[sl]), tuple(gk[sl]))
        by_type.setdefault(t, sig)
        assert by_type[t] == sig, f"copy {c} differs from its type {t}"
    assert all(int(x) == 24 or int(x) <= 24 for x in gk)
    orc = Oracle.from_aig(m.aig)
    rng = np.random.default_rng(0)
    for c in m.meta["bug_copies"]:
        sl = range(off[c], off[c + 1])
        la, lb = m.lit_a[off[c]:off[c + 1]], m.lit_b[off[c]:off[c + 1]]
        neq = [p for p in sl if gv[p] == capi.CEC_NOT_EQUIVALENT]
        for p in neq:
            hi = int(gc[p]) + 1
            if hi > (1 << 22):
                continue
            ov, oc, ok, _ = orc.check_pairs([m.lit_a[p]], [m.lit_b[p]], lo=0, hi=hi)
            assert int(ov[0]) == oracle.NOT_EQUIVALENT and int(oc[0]) == int(gc[p])
        eqs = [p for p in sl if gv[p] == capi.CEC_EQUIVALENT]
        if eqs:
            lo = int(rng.integers(0, (1 << 24) - 4096))
            ov, oc, ok, _ = orc.check_pairs(m.lit_a[eqs], m.lit_b[eqs], lo=lo, hi=lo + 4096)
            assert all(int(v) == oracle.EQUIVALENT for v in ov)
    assert any(gv == capi.CEC_NOT_EQUIVALENT)


@pytest.mark.parametrize("seed", range(20))
def test_local_checks_vs_oracle(seed):
    rng = np.random.default_rng(500 + seed)
    I = int(rng.integers(3, 12))
    m = tiny_random(I, int(rng.integers(5, 80)), 16, 500 + seed)
    N = m.aig.num_nodes
    la, lb, off, lv = [], [], [0], []
    for q in range(m.num_pairs):
        cand = rng.choice(np.arange(1, N), size=int(rng.integers(1, min(N - 1, 10) + 1)), replace=False)
        if rng.random() < 0.6:
            cand = np.unique(np.concatenate([cand, rng.choice(np.arange(1, I + 1), size=I, replace=False)]))
        cand = cand[:16]
        la.append(int(m.lit_a[q])); lb.append(int(m.lit_b[q]))
        lv += [int(x) for x in cand]
        off.append(len(lv))
    ctx = gpu_ctx(m.aig)
    got = ctx.check_local_cuts(la, lb, off, lv)
    want = Oracle.from_aig(m.aig).check_local(la, lb, off, lv)
    assert list(map(int, got)) == list(map(int, want))


@pytest.mark.parametrize("engine", ENGINES)
def test_plan_rerun_is_deterministic(engine):
    """Runs 2+ of a plan replay a captured CUDA graph (side-stream groups included); every run must
    reproduce the eager first run, which the other tests pin to the oracle."""
    for m in (c2_mul12_bug(seed=1, n=10),
              c5_big(copies=8, n_random=5, n_bugs=3, rand_pis=16, rand_ands=1500, mul_n=8)):
        ctx = gpu_ctx(m.aig, engine=engine)
        plan = capi.cec_plan_exhaustive(ctx.handle, m.lit_a, m.lit_b)
        outs = []
        for _ in range(4):
            capi.cec_plan_run(ctx.handle, plan)
            outs.append(capi.cec_plan_results(ctx.handle, plan, m.num_pairs))
        for o in outs[1:]:
            for a, b in zip(outs[0], o):
                assert np.array_equal(a, b)
        capi.cec_plan_free(plan)
        eager = gpu_ctx(m.aig, engine=engine).sim_exhaustive(m.lit_a, m.lit_b)
        for a, b in zip(eager, outs[-1]):
            assert np.array_equal(a, b)


def combine_shards(results):
    """Per-pair reduction of shard-only results (what ncclAllReduce(min) does on the device)."""
    v0 = results[0][0].copy()
    cex = np.full(v0.shape, NO, dtype=np.uint64)
    neq = np.zeros(v0.shape, bool)
    for v, c, k in results:
        hit = v == capi.CEC_NOT_EQUIVALENT
        neq |= hit
        cex = np.where(hit, np.minimum(cex, c), cex)
    v = np.where(neq, capi.CEC_NOT_EQUIVALENT, v0)
    return v, cex, results[0][2]


@pytest.mark.parametrize("world", [2, 3, 8])
@pytest.mark.parametrize("engine", SHARD_ENGINES)
def test_shard_emulation_matches_single_gpu(world, engine):
    """rank g of G simulates its slices; min over ranks == the 1-GPU result."""
    small = circuits.c3_rand(n_blocks=40, block_ands=200, num_pis=256, n_internal=300, n_near=8,
                             k_dist=((40, 10, 14),))  # windows with fewer slices than ranks: LPT owners
    for m in (c2_mul12_bug(seed=1, n=10), c5_big(copies=8, n_random=5, n_bugs=3, rand_pis=16, rand_ands=1500, mul_n=8),
              small):
        ref = gpu_ctx(m.aig, engine=engine).sim_exhaustive(m.lit_a, m.lit_b)
        parts = [gpu_ctx(m.aig, engine=engine, rank=g, world=world).sim_exhaustive(m.lit_a, m.lit_b)
                 for g in range(world)]
        v, c, k = combine_shards(parts)
        assert np.array_equal(v, ref[0]) and np.array_equal(k, ref[2])
        assert [int(x) for x, vv in zip(c, v) if vv == 2] == [int(x) for x, vv in zip(ref[1], ref[0]) if vv == 2]


def _replay_checks(res, limit=400):
    """Every logged local check of the driver, replayed through the oracle on the miter version it
    ran on: bit-exact per-check parity (the C4 outcome itself is parity-unpinned)."""
    from collections import defaultdict
    byv = defaultdict(list)
    for ch in res.checks[:limit]:
        byv[ch["version"]].append(ch)
    for vi, chs in byv.items():
        orc = Oracle.from_aig(res.versions[vi])
        off = np.cumsum([0] + [len(c["leaves"]) for c in chs])
        want = orc.check_local([c["lit_a"] for c in chs], [c["lit_b"] for c in chs], off,
                               [x for c in chs for x in c["leaves"]])
        assert [c["verdict"] for c in chs] == [int(w) for w in want]


def test_driver_dp8_local_phases_and_bug():
    from paper_conf_dac_liuy25_b200 import driver
    from workloads import c4_dp
    p = driver.CecParams(k_P=6, k_p=6, k_g=6, k_l=8, C=8)
    m = c4_dp(8)
    res = driver.check_miter(m.aig, m.lit_a, m.lit_b, p)
    assert res.checks, "local phases must run"
    _replay_checks(res)
    orc = Oracle.from_aig(m.aig)
    ov, _, _, _ = orc.check_pairs(m.lit_a, m.lit_b)
    assert all(int(v) == oracle.EQUIVALENT for v in ov)
    assert res.verdict in (capi.CEC_EQUIVALENT, capi.CEC_UNDECIDED)
    bug = c4_dp(8, bug=4)
    rb = driver.check_miter(bug.aig, bug.lit_a, bug.lit_b, p)
    ov, _, _, _ = Oracle.from_aig(bug.aig).check_pairs(bug.lit_a, bug.lit_b)
    for q in range(bug.num_pairs):  # soundness: never EQ where the oracle says NEQ
        if int(ov[q]) == oracle.NOT_EQUIVALENT:
            assert rb.po_verdicts[q] != capi.CEC_EQUIVALENT
    _replay_checks(rb)


def test_driver_c4_full():
    """C4 (BASELINE configs[3]) through the P/G/L flow with k_l = 16, C = 16: proved EQ; the bug
    variant is refuted (never EQ) and its CEX separates the PO pair in the ORIGINAL miter."""
    from paper_conf_dac_liuy25_b200 import driver
    from workloads import c4_dp
    p = driver.CecParams(k_l=16, C=16)
    m = c4_dp(64)
    res = driver.check_miter(m.aig, m.lit_a, m.lit_b, p)
    _replay_checks(res, limit=300)
    assert res.verdict == capi.CEC_EQUIVALENT, res.log[-3:]
    bug = c4_dp(64, bug=4)
    rb = driver.check_miter(bug.aig, bug.lit_a, bug.lit_b, p)
    assert rb.verdict == capi.CEC_NOT_EQUIVALENT
    orc = Oracle.from_aig(bug.aig)
    q = rb.cex_pair
    assert orc.eval_lit(int(bug.lit_a[q]), rb.cex) != orc.eval_lit(int(bug.lit_b[q]), rb.cex)
    _replay_checks(rb, limit=300)


def test_sim_patterns_and_random_classes_vs_oracle():
    """cec_sim_patterns / cec_sim_random (partial simulation for ECs): nodes get
    equal signatures iff their complement-canonical value vectors on the patterns are equal (checked
    node by node with the oracle's evaluator), and the phase bit is the node's value on pattern 0."""
    from paper_conf_dac_liuy25_b200 import driver
    m = circuits.c2_mul12_bug(seed=1, n=5)
    aig = m.aig
    ctx = gpu_ctx(aig)
    N, I = aig.num_nodes, aig.num_pis
    rng = np.random.default_rng(3)
    pats = [rng.integers(0, 2, size=I).astype(np.uint8) for _ in range(40)]
    sig, ph = capi.cec_sim_patterns(ctx.handle, N, driver.pack_patterns(pats, I))
    orc = Oracle.from_aig(aig)
    W = (len(pats) + 31) // 32 * 32  # padded patterns are all-zero assignments
    allp = pats + [np.zeros(I, np.uint8)] * (W - len(pats))
    vec = {}
    for nid in range(N):
        v = tuple(orc.eval_lit(2 * nid, p) for p in allp)
        assert int(ph[nid]) == v[0]
        vec[nid] = tuple(x ^ v[0] for x in v)
    for a in range(N):
        for b in range(a + 1, N, 7):
            assert (int(sig[a]) == int(sig[b])) == (vec[a] == vec[b])


def test_nccl_min_allreduce_single_rank():
    """The NCCL path of a10 on one GPU: a 1-rank communicator from cec_nccl_unique_id, the min
    all-reduce runs inside cec_plan_run and the results equal the no-NCCL run."""
    m = c2_mul12_bug(seed=1, n=10)
    uid = capi.cec_nccl_unique_id()
    got = gpu_ctx(m.aig, rank=0, world=1, nccl_unique_id=uid).sim_exhaustive(m.lit_a, m.lit_b)
    ref = gpu_ctx(m.aig).sim_exhaustive(m.lit_a, m.lit_b)
    for a, b in zip(got, ref):
        assert np.array_equal(a, b)


@pytest.mark.parametrize("case", range(8))
def test_gpu_cut_generator_matches_cut_oracle(case):
    """NEXT-1: the GPU cut generator (level-parallel by Eq. 2, warp per node) returns exactly the cuts
    of oracle/cuts.py (Eq. 1 + Table I + dominance + similarity, exact arithmetic)."""
    from oracle import cuts as cut_oracle
    from workloads import c4_dp
    rng = np.random.default_rng(50 + case)
    m = c4_dp(6 + 2 * case) if case < 4 else circuits.random_miter(12, 150 + 60 * case, 10, seed=950 + case, window=24)
    aig = m.aig
    pairs = set()
    for a, b in zip(m.lit_a, m.lit_b):
        x, y = sorted((int(a) >> 1, int(b) >> 1))
        if x < y:
            pairs.add((x, y))
    for _ in range(30):
        x, y = sorted(int(v) for v in rng.integers(1, aig.num_nodes, size=2))
        if x < y:
            pairs.add((x, y))
    seen, P = set(), []
    for x, y in sorted(pairs):
        if y not in seen:
            seen.add(y)
            P.append((x, y))
    k_l, C, pass_id, mc = int(rng.integers(4, 17)), int(rng.integers(2, 17)), case % 3, int(rng.integers(1, 9))
    ctx = gpu_ctx(aig)
    os.environ["CEC_CUTS_GPU"] = "1"  # small cones would otherwise use the host generator
    try:
        pco, co, lv = capi.cec_common_cuts(ctx.handle, [x for x, _ in P], [y for _, y in P], k_l, C, pass_id, mc)
    finally:
        del os.environ["CEC_CUTS_GPU"]
    want = cut_oracle.common_cuts(aig.num_pis, aig.fanins, [x for x, _ in P], [y for _, y in P], k_l, C, pass_id, mc)
    for i in range(len(P)):
        got = [tuple(int(v) for v in lv[co[t]:co[t + 1]]) for t in range(int(pco[i]), int(pco[i + 1]))]
        assert got == want[i], (i, P[i], got, want[i])


@pytest.mark.parametrize("k_max", [8, 16, 32])
def test_gpu_supports_match_host_walk(k_max, monkeypatch):
    """a2 on the device (supp_gpu.cu, lists saturating at k_max + 1) gives the same k, verdicts and
    CEX as the host cone walk, including pairs above k_max (exact k recomputed on the host)."""
    from workloads import c4_dp

    saturated = False
    for m in (c4_dp(16), c5_big(copies=6, n_random=4, n_bugs=3, rand_pis=14, rand_ands=700, mul_n=7)):
        outs = []
        for flag in ("0", "1"):
            monkeypatch.setenv("CEC_SUPP_GPU", flag)
            outs.append(gpu_ctx(m.aig, k_max=k_max, merge=capi.CEC_MERGE_PAPER).sim_exhaustive(m.lit_a, m.lit_b))
        for a, b in zip(*outs):
            assert np.array_equal(a, b)
        saturated |= bool((outs[0][2] > k_max).any())
    assert saturated  # the saturated-list path (host re-walk) was exercised


@pytest.mark.parametrize("engine", ENGINES)
def test_pipelined_call_matches_single_plan(engine, monkeypatch):
    """cec_sim_exhaustive cuts the merged windows into chunks planned/launched in a pipeline
    (CEC_PIPELINE); any chunking must give the single-plan results (verdict, CEX, k)."""
    m = c5_big(copies=12, n_random=6, n_bugs=4, rand_pis=14, rand_ands=900, mul_n=7)
    ctx = gpu_ctx(m.aig, engine=engine)
    plan = capi.cec_plan_exhaustive(ctx.handle, m.lit_a, m.lit_b)
    capi.cec_plan_run(ctx.handle, plan)
    ref = capi.cec_plan_results(ctx.handle, plan, m.num_pairs)
    capi.cec_plan_free(plan)
    assert (ref[0] == capi.CEC_NOT_EQUIVALENT).any()
    for K in ("1", "2", "3", "5", "64"):
        monkeypatch.setenv("CEC_PIPELINE", K)
        got = ctx.sim_exhaustive(m.lit_a, m.lit_b)
        for a, b in zip(ref, got):
            assert np.array_equal(a, b), K
        orc = Oracle.from_aig(m.aig)
        for p in np.flatnonzero(got[0] == capi.CEC_NOT_EQUIVALENT)[:3]:
            pis = ctx.get_cex(int(p))  # the CEX vector of the pipelined call distinguishes the pair
            assert orc.eval_lit(int(m.lit_a[p]), pis) != orc.eval_lit(int(m.lit_b[p]), pis)


def _c3_small():
    """A reduced C3: 30 random blocks with supports 10..16 over 256 PIs (oracle in seconds) — many
    distinct small window structures, i.e. the JIT bundle kernels (jit_source_bundle)."""
    return circuits.c3_rand(n_blocks=30, block_ands=300, num_pis=256, n_internal=600, n_near=32,
                            k_dist=((30, 10, 16),))


def test_jit_bundles_vs_oracle_and_unbundled(monkeypatch):
    m = _c3_small()
    ctx, gv, gc, gk = check_vs_oracle(m, engine=capi.CEC_ENGINE_JIT, merge=capi.CEC_MERGE_COST)
    st = ctx.stats()
    assert st["jit_windows"] > st["jit_kernels"]  # structures were bundled
    monkeypatch.setenv("CEC_NO_BUNDLE", "1")
    ctx2 = gpu_ctx(m.aig, engine=capi.CEC_ENGINE_JIT, merge=capi.CEC_MERGE_COST)
    got = ctx2.sim_exhaustive(m.lit_a, m.lit_b)
    for a, b in zip((gv, gc, gk), got):
        assert np.array_equal(a, b)
    monkeypatch.setenv("CEC_BUNDLE_MAX", "3")
    monkeypatch.delenv("CEC_NO_BUNDLE")
    ctx3 = gpu_ctx(m.aig, engine=capi.CEC_ENGINE_JIT, merge=capi.CEC_MERGE_COST)
    got = ctx3.sim_exhaustive(m.lit_a, m.lit_b)
    for a, b in zip((gv, gc, gk), got):
        assert np.array_equal(a, b)


def test_split_pipeline_vs_oracle(monkeypatch, capfd):
    """Many small windows: the public call plans and launches the large windows (estimated sweep
    >= CEC_PIPE_SPLIT node-words) as a first chunk and the rest while they run. Any split point
    gives the oracle's results (verdicts, k, CEX indices); at least one threshold really splits."""
    m = _c3_small()
    orc = Oracle.from_aig(m.aig)
    ov, oc, ok, _ = orc.check_pairs(m.lit_a, m.lit_b, k_max=32)
    monkeypatch.setenv("CEC_TIMING", "1")
    monkeypatch.setenv("CEC_PIPE_SPLIT_MINWIN", "8")
    splits = 0
    for e in range(6, 20, 2):
        monkeypatch.setenv("CEC_PIPE_SPLIT", str(float(2 ** e)))
        ctx = gpu_ctx(m.aig, merge=capi.CEC_MERGE_COST)
        gv, gc, gk = ctx.sim_exhaustive(m.lit_a, m.lit_b)
        assert_same(gv, gc, gk, ov, oc, ok, f"split 2^{e}")
        for p in np.nonzero(gv == capi.CEC_NOT_EQUIVALENT)[0][:8]:
            vec = ctx.get_cex(int(p))
            assert orc.eval_lit(int(m.lit_a[p]), vec) != orc.eval_lit(int(m.lit_b[p]), vec)
        splits += "call: split" in capfd.readouterr().err
    assert splits >= 1


def test_c5_full_vs_stored_oracle():
    """Full-size C5 (2.1M ANDs, 6320 pairs, 256 windows x 2^24 patterns) in the launch
    configuration bench.py times, against the oracle's result for EVERY pair
    (tests/golden/c5_big.json, scripts/make_golden_c5.py: one single-threaded oracle task per copy)."""
    g = _golden("c5_big")
    m = c5_big()
    assert [int(x) for x in m.lit_a] == g["lit_a"] and [int(x) for x in m.lit_b] == g["lit_b"]
    ctx = gpu_ctx(m.aig)
    plan = capi.cec_plan_exhaustive(ctx.handle, m.lit_a, m.lit_b)
    capi.cec_plan_run(ctx.handle, plan)
    gv, gc, gk = capi.cec_plan_results(ctx.handle, plan, m.num_pairs)
    capi.cec_plan_free(plan)
    assert_same(gv, gc, gk, np.array(g["verdict"]), np.array([int(x) for x in g["cex"]], dtype=np.uint64),
                np.array(g["k"]), "c5 full")
    orc = Oracle.from_aig(m.aig)
    for p in np.nonzero(gv == capi.CEC_NOT_EQUIVALENT)[0]:  # each CEX really separates the pair
        want = orc.cex_vector(int(m.lit_a[p]), int(m.lit_b[p]), int(gc[p]))
        assert orc.eval_lit(int(m.lit_a[p]), want) != orc.eval_lit(int(m.lit_b[p]), want)


def test_c3_full_vs_stored_oracle():
    """Full-size C3 (234k ANDs, 6664 pairs incl. 64 near-miss NEQ pairs, supports up to 29) in the
    launch configuration bench.py times (cost-aware merge, AUTO engine: JIT bundles + interpreter),
    against the oracle's result for EVERY pair (tests/golden/c3_rand.json, scripts/make_golden_c3.py:
    support groups x pattern ranges, min-reduced)."""
    from workloads import c3_rand

    g = _golden("c3_rand")
    m = c3_rand()
    assert [int(x) for x in m.lit_a] == g["lit_a"] and [int(x) for x in m.lit_b] == g["lit_b"]
    ctx = gpu_ctx(m.aig, merge=capi.CEC_MERGE_COST)
    plan = capi.cec_plan_exhaustive(ctx.handle, m.lit_a, m.lit_b)
    capi.cec_plan_run(ctx.handle, plan)
    gv, gc, gk = capi.cec_plan_results(ctx.handle, plan, m.num_pairs)
    capi.cec_plan_free(plan)
    assert_same(gv, gc, gk, np.array(g["verdict"]), np.array([int(x) for x in g["cex"]], dtype=np.uint64),
                np.array(g["k"]), "c3 full")
    assert (gv == capi.CEC_NOT_EQUIVALENT).sum() >= 1
    ve, ce, ke = ctx.sim_exhaustive(m.lit_a, m.lit_b)  # the pipelined public call agrees
    assert np.array_equal(ve, gv) and np.array_equal(ke, gk)
    assert np.array_equal(ce[gv == capi.CEC_NOT_EQUIVALENT], gc[gv == capi.CEC_NOT_EQUIVALENT])


@pytest.mark.parametrize("mode", ["0", "1", "2", "3"])
def test_jit_cell_mappings_vs_oracle(mode, monkeypatch):
    """Every cell mapping of the JIT body (0: one LOP3 per AND, 1: greedy fusion, 2: area-flow
    3-LUTs, 3: 3-LUTs + IMAD cells on the FMA pipe, the default) gives the oracle's verdicts, k and
    canonical CEX indices bit for bit: a multiplier with an injected bug (NEQ, early exit), a
    reduced C5 (word-uniform masks from inputs and nodes) and C3-style random windows."""
    monkeypatch.setenv("CEC_JIT_FUSE", mode)
    for m in (c2_mul12_bug(seed=1, n=10), c5_big(copies=6, n_random=4, n_bugs=2, rand_pis=18, rand_ands=1200, mul_n=9),
              circuits.random_miter(20, 900, 12, seed=77, window=40)):
        ctx, gv, gc, gk = check_vs_oracle(m, engine=capi.CEC_ENGINE_JIT)
        st = ctx.stats()
        assert st["jit_windows"] >= 1
        assert (st["imad_words"] > 0) == (mode == "3") or m.name.startswith("rand")
        ctx.close()


@pytest.mark.parametrize("seed", range(24))
def test_fuzz_jit_windows_word_uniform_inputs(seed):
    """JIT windows at the input positions where the dual-pipe cells change: k = 10..14 (inputs 0..4
    per-bit masks, 5..9 lane-uniform, >= 10 slice-uniform words), random AIGs whose ANDs read PIs
    often (many IMAD candidates: AND of a PI or of a node over PIs >= 5 with anything), random
    pair literals including complemented and constant ones; JIT engine vs the oracle, bit for bit."""
    rng = np.random.default_rng(500 + seed)
    I = int(rng.integers(10, 15))
    m = tiny_random(I, int(rng.integers(40, 260)), 20, 9000 + seed)
    ctx, gv, gc, gk = check_vs_oracle(m, k_max=14, merge=int(rng.integers(0, 3)), engine=capi.CEC_ENGINE_JIT)
    ctx.close()


@pytest.mark.parametrize("seed", range(8))
def test_local_checks_jit_engine_vs_oracle(seed):
    """a12 local checks through the JIT register kernels (engine forced): cut leaves are the window
    inputs, so leaves 5.. are word-uniform words and feed the IMAD cells exactly like PIs do;
    random cuts of 10..16 leaves (valid or not: invalid cuts must come back CEC_E_CUT-marked the
    same way) against the oracle's local check."""
    rng = np.random.default_rng(900 + seed)
    I = int(rng.integers(10, 15))
    m = tiny_random(I, int(rng.integers(60, 200)), 12, 900 + seed)
    N = m.aig.num_nodes
    la, lb, off, lv = [], [], [0], []
    for q in range(m.num_pairs):
        cand = rng.choice(np.arange(1, N), size=int(rng.integers(4, 12)), replace=False)
        cand = np.unique(np.concatenate([cand, np.arange(1, I + 1)]))[:16]  # PIs make most cuts valid
        la.append(int(m.lit_a[q])); lb.append(int(m.lit_b[q]))
        lv += [int(x) for x in cand]
        off.append(len(lv))
    ctx = gpu_ctx(m.aig, engine=capi.CEC_ENGINE_JIT)
    got = ctx.check_local_cuts(la, lb, off, lv)
    want = Oracle.from_aig(m.aig).check_local(la, lb, off, lv)
    assert list(map(int, got)) == list(map(int, want))
    ctx.close()


def test_reload_aig_matches_fresh_context_and_oracle():
    """cec_reload_aig (include/cec.h): a device context reloaded with the next miter gives exactly
    the oracle's results for it (and a fresh context's), with no state of the previous AIG left:
    its per-node support table, device AIG copy and last CEX are dropped."""
    a = circuits.c2_mul12_bug(seed=1, n=8)
    b = c5_big(copies=6, n_random=4, n_bugs=2, rand_pis=14, rand_ands=800, mul_n=7)
    ctx = gpu_ctx(a.aig)
    va, ca, ka = ctx.sim_exhaustive(a.lit_a, a.lit_b)
    assert (va == capi.CEC_NOT_EQUIVALENT).any()
    ctx.reload(b.aig, k_max=32)
    with pytest.raises(capi.CecError) as e:  # the last check belonged to the old AIG
        ctx.get_cex(int(np.nonzero(va == capi.CEC_NOT_EQUIVALENT)[0][0]))
    assert e.value.status == capi.CEC_E_STATE
    got = ctx.sim_exhaustive(b.lit_a, b.lit_b)
    orc = Oracle.from_aig(b.aig)
    ov, oc, ok, _ = orc.check_pairs(b.lit_a, b.lit_b, k_max=32)
    assert_same(*got, ov, oc, ok, "reloaded")
    for x, y in zip(got, gpu_ctx(b.aig).sim_exhaustive(b.lit_a, b.lit_b)):
        assert np.array_equal(x, y)
    ctx.reload(a.aig)  # and back: the first AIG's results again
    for x, y in zip(ctx.sim_exhaustive(a.lit_a, a.lit_b), (va, ca, ka)):
        assert np.array_equal(x, y)


def test_plan_sweep_timing_events():
    """cec_plan_sweep_timing / cec_plan_sweep_ms (include/cec.h): off by default (CEC_E_STATE), on:
    the window kernels' event interval of the last run, positive and inside the run's own events,
    also across a CUDA-graph replay; results are unchanged by the extra event nodes."""
    m = c5_big(copies=6, n_random=4, n_bugs=2, rand_pis=14, rand_ands=800, mul_n=7)
    ctx = gpu_ctx(m.aig)
    plan = capi.cec_plan_exhaustive(ctx.handle, m.lit_a, m.lit_b)
    capi.cec_plan_run(ctx.handle, plan)
    ref = capi.cec_plan_results(ctx.handle, plan, m.num_pairs)
    with pytest.raises(capi.CecError) as e:
        capi.cec_plan_sweep_ms(plan)
    assert e.value.status == capi.CEC_E_STATE
    capi.cec_plan_sweep_timing(plan, True)
    for _ in range(3):  # direct launch, capture, replay
        capi.cec_plan_run(ctx.handle, plan)
        got = capi.cec_plan_results(ctx.handle, plan, m.num_pairs)
        for a, b in zip(ref, got):
            assert np.array_equal(a, b)
        sw = capi.cec_plan_sweep_ms(plan)
        assert 0.0 < sw <= ctx.stats()["kernel_ms"] + 1e-3
    capi.cec_plan_sweep_timing(plan, False)
    capi.cec_plan_run(ctx.handle, plan)
    capi.cec_plan_results(ctx.handle, plan, m.num_pairs)
    with pytest.raises(capi.CecError):
        capi.cec_plan_sweep_ms(plan)
    capi.cec_plan_free(plan)


@pytest.mark.parametrize("world", [2, 3])
def test_shard_emulation_with_split_pipeline(world, monkeypatch):
    """Pattern-space shards (rank g of G, shard-only mode) through the public call with the
    large-windows-first split forced: the min over ranks is still the 1-GPU result."""
    m = _c3_small()
    ref = gpu_ctx(m.aig, merge=capi.CEC_MERGE_COST).sim_exhaustive(m.lit_a, m.lit_b)
    monkeypatch.setenv("CEC_PIPE_SPLIT", str(float(1 << 12)))
    monkeypatch.setenv("CEC_PIPE_SPLIT_MINWIN", "2")
    parts = [gpu_ctx(m.aig, merge=capi.CEC_MERGE_COST, rank=g, world=world).sim_exhaustive(m.lit_a, m.lit_b)
             for g in range(world)]
    v, c, k = combine_shards(parts)
    assert np.array_equal(v, ref[0]) and np.array_equal(k, ref[2])
    neq = ref[0] == capi.CEC_NOT_EQUIVALENT
    assert neq.any() and np.array_equal(np.asarray(c)[neq], ref[1][neq])


@pytest.mark.parametrize("kib", [64, 256, 4096])
def test_simt_engine_caller_workspace(kib):
    """cec_opts.workspace (include/cec.h): the paper's Alg. 1 engine sizes E from the caller's memory
    budget M and keeps its simulation table in the caller's device buffer; a small M
    means more rounds (E words per row per round), never different results."""
    m = circuits.c2_mul12_bug(seed=1, n=8)
    ws = torch.empty(kib * 1024, dtype=torch.uint8, device="cuda")
    ctx = gpu_ctx(m.aig, engine=capi.CEC_ENGINE_SIMT, workspace=ws.data_ptr(), workspace_bytes=ws.numel())
    got = ctx.sim_exhaustive(m.lit_a, m.lit_b)
    orc = Oracle.from_aig(m.aig)
    ov, oc, ok, _ = orc.check_pairs(m.lit_a, m.lit_b, k_max=32)
    assert_same(*got, ov, oc, ok, f"simt workspace {kib} KiB")
    ref = gpu_ctx(m.aig, engine=capi.CEC_ENGINE_SIMT).sim_exhaustive(m.lit_a, m.lit_b)
    for a, b in zip(got, ref):
        assert np.array_equal(a, b)


def test_cli_diffable_output_matches_oracle_byte_for_byte(tmp_path):
    """SURVEY.md §8(c) "Diffable output": the GPU path's CLI and the oracle's CLI, given the same
    AIGER, pair and check files, print byte-identical text (verdicts, k, CEX indices, CEX vectors;
    local checks)."""
    import subprocess
    import sys as _sys

    from workloads import write_aag, write_checks, write_pairs

    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    m = circuits.c2_mul12_bug(seed=3, n=8)
    write_aag(m.aig, str(tmp_path / "m.aag"))
    write_pairs(str(tmp_path / "p.txt"), m.lit_a, m.lit_b)
    orc = Oracle.from_aig(m.aig)
    off, lv = [0], []
    for a, b in zip(m.lit_a, m.lit_b):  # cut = the pair's support (local verdict = global)
        s = orc.support(int(a), int(b))
        lv += s
        off.append(len(lv))
    write_checks(str(tmp_path / "c.txt"), m.lit_a, m.lit_b, off, lv)
    outs = {}
    for cmd, f in (("check", "p.txt"), ("local", "c.txt")):
        want = oracle.run_cli(cmd, str(tmp_path / "m.aag"), str(tmp_path / f))
        got = subprocess.run([_sys.executable, "-m", "paper_conf_dac_liuy25_b200.cli", cmd, str(tmp_path / "m.aag"),
                              str(tmp_path / f)], capture_output=True, text=True, cwd=root, timeout=300)
        assert got.returncode == 0, got.stderr[-2000:]
        assert got.stdout == want, cmd
        outs[cmd] = want
    assert " NEQ " in outs["check"] and "\ncex " in outs["check"]  # the bug is refuted, with a CEX line


@pytest.mark.parametrize("which", ["small", "full", "bigcones"])
def test_gpu_cone_sizes_give_the_host_merge(which, monkeypatch):
    """The cost-aware merge's cone sizes from the GPU walk (supp_gpu.cu cone_sizes) equal the host
    walk's: the merged windows (inputs, node counts, pairs) and W are identical to the host-walk
    plan (CEC_CONES_GPU=0), and so are the results."""
    from workloads import c3_rand

    if which == "bigcones":  # 10k-AND copies: cones beyond the kernel's shared memory -> host fallback
        m = c5_big(copies=8, n_random=6, n_bugs=2)
    else:
        m = _c3_small() if which == "small" else c3_rand()

    def plan_of():
        ctx = gpu_ctx(m.aig, merge=capi.CEC_MERGE_COST, engine=capi.CEC_ENGINE_INTERP)
        pl = capi.cec_plan_exhaustive(ctx.handle, m.lit_a, m.lit_b)
        info = capi.cec_plan_info(pl)
        wins = [capi.cec_plan_window(pl, w) for w in range(info["num_windows"])]
        capi.cec_plan_run(ctx.handle, pl)
        res = capi.cec_plan_results(ctx.handle, pl, m.num_pairs)
        capi.cec_plan_free(pl)
        return info, wins, res

    gi, gw, gr = plan_of()
    monkeypatch.setenv("CEC_CONES_GPU", "0")
    hi, hw, hr = plan_of()
    assert gi == hi and gw == hw
    for a, b in zip(gr, hr):
        assert np.array_equal(a, b)
