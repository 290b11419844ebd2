"""Host driver above the C ABI: the simulation-based CEC flow of PAPER.md §III-D (Fig. 5, :179-187).

  P phase  PO pairs with support <= k_P (all) or <= k_p (subset) -> cec_sim_exhaustive
  ECs partial simulation of random + CEX patterns and exact classes on the
            GPU (cec_sim_classes) -> pairs (repr = minimum id, member, phase)
  G phase  candidate pairs with support <= k_g -> cec_sim_exhaustive
  L phases  (§III-C) 3 passes of cut enumeration (Eq. 1, Table I orders) and local
            checks (cec_check_local_cuts); reduce the miter after each phase; repeat until no progress
  reduction proved pairs are merged (member -> representative) and the miter is
            rebuilt with structural hashing on the GPU (cec_reduce)

Every simulation, the class formation and the miter rebuild run in libcec.so's CUDA kernels; cuts
come from the native cut generator (cec_common_cuts, GPU for large cones). The host part here is
the phase policy and its bookkeeping. Undecided pairs remain undecided (the paper
then hands the reduced miter to ABC, which is out of scope).
"""
from __future__ import annotations

import atexit
import bisect
import collections.abc
import dataclasses
import gc
import time
from typing import Dict, List, Optional, Tuple

import numpy as np

from . import capi
from workloads.aig import Aig  # plain container (num_pis, fanins, pos); no graph building here


@dataclasses.dataclass
class CecParams:
    k_P: int = 32
    k_p: int = 16
    k_g: int = 16
    k_l: int = 8
    C: int = 8
    sim_words: int = 64    # random patterns = 32 * sim_words
    seed: int = 1
    max_phases: int = 64
    max_cuts_per_pair: int = 8
    final_po_check: bool = True  # after the L phases: exhaustive check of undecided POs with k <= k_P
    native_cuts: bool = True     # C++ cut generator (cec_common_cuts); False = the Python reference
    max_cex_patterns: int = 1024  # CEX patterns kept for class refinement
    buffer_checks: int = 4096     # Alg. 2 common-cut buffer (local checks per flush)
    distance1: bool = True        # also simulate every distance-1 neighbour of each CEX
    device: int = 0
    engine: int = capi.CEC_ENGINE_AUTO
    reuse_context: bool = True    # keep the device context(s) for the next check_miter call


class CheckLog(collections.abc.Sequence):
    """Replay log of every local check (SURVEY.md §5 "checkpoint / resume": the oracle re-checks
    each (miter version, pair, cut) and its verdict). Kept as the per-pass arrays the native pass
    returns; entries are dicts {version, phase, pass, lit_a, lit_b, leaves, verdict} made on access
    (building 57k dicts inside the flow cost ~20% of C4's end-to-end time)."""

    def __init__(self):
        self._chunks = []  # (version, phase, pass, lit_a[], lit_b[], cut_off[], leaves[], verdict[])
        self._starts = [0]

    def add(self, version, phase, pass_id, lit_a, lit_b, cut_off, leaves, verdict) -> None:
        n = len(lit_a)
        if n:
            self._chunks.append((version, phase, pass_id, np.array(lit_a), np.array(lit_b), np.array(cut_off),
                                 np.array(leaves), np.array(verdict)))  # copies: the pass's buffers are larger
            self._starts.append(self._starts[-1] + n)

    def append(self, ch: dict) -> None:
        self.add(ch["version"], ch["phase"], ch["pass"], [ch["lit_a"]], [ch["lit_b"]], [0, len(ch["leaves"])],
                 list(ch["leaves"]), [ch["verdict"]])

    def __len__(self) -> int:
        return self._starts[-1]

    def _entry(self, k: int, i: int) -> dict:
        v, ph, pa, la, lb, off, lv, vd = self._chunks[k]
        return {"version": v, "phase": ph, "pass": pa, "lit_a": int(la[i]), "lit_b": int(lb[i]),
                "leaves": [int(x) for x in lv[off[i]:off[i + 1]]], "verdict": int(vd[i])}

    def __getitem__(self, idx):
        if isinstance(idx, slice):
            return [self[i] for i in range(*idx.indices(len(self)))]
        if idx < 0:
            idx += len(self)
        if not 0 <= idx < len(self):
            raise IndexError(idx)
        k = bisect.bisect_right(self._starts, idx) - 1
        return self._entry(k, idx - self._starts[k])

    def __iter__(self):
        for k, ch in enumerate(self._chunks):
            for i in range(len(ch[3])):
                yield self._entry(k, i)


@dataclasses.dataclass
class CecResult:
    verdict: int                      # CEC_EQUIVALENT / CEC_NOT_EQUIVALENT / CEC_UNDECIDED
    po_verdicts: np.ndarray
    cex: Optional[np.ndarray] = None  # PI values (PI id i+1 = cex[i]) of the lowest NEQ PO pair
    cex_pair: int = -1
    log: List[dict] = dataclasses.field(default_factory=list)
    checks: "CheckLog" = dataclasses.field(default_factory=lambda: CheckLog())  # replay log of every local check
    versions: List[Aig] = dataclasses.field(default_factory=list)  # miter versions the checks refer to
    final_ands: int = 0


# ---------------------------------------------------------------------------------------------
# miter bookkeeping
# ---------------------------------------------------------------------------------------------

class Miter:
    """Current (reduced) miter: an AIG plus the PO pair literals expressed in it."""

    def __init__(self, aig: Aig, lit_a, lit_b):
        self.aig = aig
        self.lit_a = np.asarray(lit_a, dtype=np.uint32).copy()
        self.lit_b = np.asarray(lit_b, dtype=np.uint32).copy()

    def reduce(self, subst: Dict[int, int], device: int = 0,
               ctx: Optional[capi.Context] = None) -> Tuple["Miter", np.ndarray]:
        """Merge proved pairs: node id -> literal of its (lower-id) representative,
        rebuilt with structural hashing so merged fanouts collapse — on the GPU (cec_reduce), with
        `ctx` (a device context of this miter's AIG) or a temporary one.
        Returns the reduced miter and the image (new literal) of every old node id."""
        own = ctx is None
        if own:
            ctx = capi.Context.from_aig(self.aig, device=device)
        try:
            mem = np.fromiter(subst.keys(), dtype=np.uint32, count=len(subst))
            rep = np.fromiter(subst.values(), dtype=np.uint32, count=len(subst))
            fan, image, lits = ctx.reduce(mem, rep, np.concatenate([self.lit_a, self.lit_b]))
        finally:
            if own:
                ctx.close()
        P = self.lit_a.size
        aig = Aig(self.aig.num_pis, np.ascontiguousarray(fan, dtype=np.uint32), lits.astype(np.uint32))
        return Miter(aig, lits[:P], lits[P:]), image


def _remap_tried(tried, image: np.ndarray):
    """(repr, member, phase) tuples of one miter version -> the same functional pairs in the reduced
    version, whose node ids are renumbered (cec_reduce). `image[id]` = new literal of old node id.
    A pair whose two sides collapsed into one node is dropped (nothing left to decide)."""
    out = set()
    for r, m_, f in tried:
        a, b = int(image[r]), int(image[m_]) ^ f
        if a >> 1 == b >> 1:
            continue
        lo, hi = (a, b) if (a >> 1) < (b >> 1) else (b, a)
        out.add((lo >> 1, hi >> 1, (a ^ b) & 1))
    return out


def _ctx(aig: Aig, p: CecParams, k_max: int, k_s: Optional[int] = None) -> capi.Context:
    return capi.Context.from_aig(aig, device=p.device, k_max=k_max, k_s=k_s or k_max, engine=p.engine)


# ---------------------------------------------------------------------------------------------
# cut enumeration (Eq. 1) with Table I selection — host-minimal
# ---------------------------------------------------------------------------------------------

def _bits(mask: int) -> List[int]:
    out = []
    while mask:
        low = mask & -mask
        out.append(low.bit_length() - 1)
        mask ^= low
    return out


def enumerate_cuts(aig: Aig, k_l: int, C: int, pass_id: int, repr_of: Optional[Dict[int, int]] = None
                   ) -> List[List[int]]:
    """P(n) for every node id as bitmasks over node ids. E(n) = {u | v : u in P(n0) + {{n0}},
    v in P(n1) + {{n1}}, |u | v| <= k_l} (Eq. 1); P(n) = the C best of E(n) under the
    Table I order of this pass: pass 1 fanout > size > small level; pass 2 small
    level > size > fanout; pass 3 large level > size > fanout. PIs: P = {{pi}} (Alg. 2 l.4-5).
    Dominated cuts (supersets of another candidate) are dropped first (priority cuts, ref. [27]).
    Similarity-guided selection: for a non-representative n (repr_of[n] = r) the
    candidates are ranked first by s(c, P(r)) = sum_{c' in P(r)} |c & c'| / |c | c'| (larger
    first), then by the Table I order. Ids ascend, so P(r) is ready before P(n) (r < n), which is
    what the enumeration levels of Eq. (2) guarantee in the paper's level-wise schedule."""
    I, A = aig.num_pis, aig.num_ands
    N = 1 + I + A
    fan = aig.fanins.astype(np.int64)
    level = np.zeros(N, dtype=np.int64)
    fanout = np.zeros(N, dtype=np.int64)
    for j in range(A):
        a, b = int(fan[j, 0]) >> 1, int(fan[j, 1]) >> 1
        level[1 + I + j] = 1 + max(level[a], level[b])
        fanout[a] += 1
        fanout[b] += 1
    P: List[List[int]] = [[] for _ in range(N)]
    for i in range(1, I + 1):
        P[i] = [1 << i]
    P[0] = [1]  # constant: treat as its own leaf
    repr_of = repr_of or {}

    def key(mask: int):
        ids = _bits(mask)
        sz = len(ids)
        avg_f = sum(int(fanout[x]) for x in ids) / sz
        avg_l = sum(int(level[x]) for x in ids) / sz
        if pass_id == 0:
            return (-avg_f, sz, avg_l)
        if pass_id == 1:
            return (avg_l, sz, -avg_f)
        return (-avg_l, sz, -avg_f)

    for j in range(A):
        n = 1 + I + j
        a, b = int(fan[j, 0]) >> 1, int(fan[j, 1]) >> 1
        ua = P[a] + [1 << a]
        vb = P[b] + [1 << b]
        E = set()
        for u in ua:
            for v in vb:
                c = u | v
                if c.bit_count() <= k_l:
                    E.add(c)
        E.discard(1 << n)
        # drop dominated cuts (a proper superset of another candidate)
        Es = sorted(E, key=lambda x: x.bit_count())
        kept: List[int] = []
        for c in Es:
            if not any((c & d) == d for d in kept):
                kept.append(c)
        r = repr_of.get(n)
        if r is not None and P[r]:
            Pr = P[r]
            P[n] = sorted(kept, key=lambda c: (-sum((c & d).bit_count() / (c | d).bit_count() for d in Pr),) + key(c))[:C]
        else:
            P[n] = sorted(kept, key=key)[:C]
    return P


# ---------------------------------------------------------------------------------------------
# the flow
# ---------------------------------------------------------------------------------------------

def pack_patterns(patterns: List[np.ndarray], num_pis: int) -> np.ndarray:
    """Pack PI assignments (uint8[num_pis] each) into u32 words: pattern j is bit j%32 of word j//32."""
    W = max(1, (len(patterns) + 31) // 32)
    words = np.zeros((num_pis, W), dtype=np.uint32)
    for j, pat in enumerate(patterns):
        words[:, j // 32] |= (np.asarray(pat[:num_pis], dtype=np.uint32) & 1) << np.uint32(j % 32)
    return words


def check_miter(aig: Aig, lit_a, lit_b, params: Optional[CecParams] = None) -> CecResult:
    p = params or CecParams()
    cur = Miter(aig, lit_a, lit_b)
    log: List[dict] = []
    checks = CheckLog()
    versions: List[Aig] = []
    P = cur.lit_a.size
    po_v = np.full(P, capi.CEC_UNDECIDED, dtype=np.int32)

    def po_status(m: Miter):
        return np.array([capi.CEC_EQUIVALENT if a == b else capi.CEC_UNDECIDED for a, b in zip(m.lit_a, m.lit_b)],
                        dtype=np.int32)

    # One device context serves every phase: each new miter version is loaded into it
    # (cec_reload_aig), keeping streams, workers, device pools and JIT kernels.
    # A second one (slot 1) holds the local-check limit when k_l > k_g. With reuse_context the
    # contexts also outlive the call (release_contexts() frees them): the next miter is loaded into
    # them instead of creating contexts and freeing their device memory per call (context creation
    # is excluded from end-to-end time; cudaFree of a pool can take 0.3 s).
    dev: List[Optional[capi.Context]] = (_DEV_CACHE.setdefault((p.device, p.engine), [None, None])
                                         if p.reuse_context else [None, None])

    def dctx(m: Miter, k_max: int, slot: int = 0) -> capi.Context:
        if dev[slot] is None:
            dev[slot] = _ctx(m.aig, p, k_max)
        else:
            dev[slot].reload(m.aig, k_max=k_max)
        return dev[slot]

    # The flow allocates only acyclic records (tens of thousands of per-check entries), which
    # reference counting frees; the cyclic collector's full passes over them cost 0.1-0.3 s spikes
    # in random phases, so it is paused for the flow and restored afterwards.
    gc_was_on = gc.isenabled()
    gc.disable()
    ok = False
    try:
        res = _flow(p, cur, log, checks, versions, P, po_v, po_status, dctx)
        ok = True
        return res
    finally:
        if not p.reuse_context or not ok:  # a failed flow does not leave its contexts for the next
            for i, c in enumerate(dev):
                if c is not None:
                    c.close()
                    dev[i] = None
        if gc_was_on:
            gc.enable()


# device contexts kept between check_miter calls, per (device, engine); one caller thread at a time
_DEV_CACHE: Dict[Tuple[int, int], List[Optional[capi.Context]]] = {}


def release_contexts() -> None:
    """Free the device contexts check_miter keeps between calls (reuse_context)."""
    for slots in _DEV_CACHE.values():
        for i, c in enumerate(slots):
            if c is not None:
                c.close()
                slots[i] = None
    _DEV_CACHE.clear()


atexit.register(release_contexts)  # before the CUDA runtime's own teardown (registered earlier)


def _flow(p, cur, log, checks, versions, P, po_v, po_status, dctx) -> CecResult:
    # ---- P phase -------------------------------------------------------------
    t = time.perf_counter()
    hctx = capi.Context.from_aig(cur.aig, device=-1, k_max=63)
    ks = np.array([hctx.pair_k(int(a), int(b)) for a, b in zip(cur.lit_a, cur.lit_b)])
    hctx.close()
    thr = p.k_P if (ks <= p.k_P).all() else p.k_p
    sel = np.nonzero(ks <= thr)[0]
    subst: Dict[int, int] = {}
    ctx = None
    if sel.size:
        ctx = dctx(cur, thr)
        v, cex, k = ctx.sim_exhaustive(cur.lit_a[sel], cur.lit_b[sel])
        for i, q in enumerate(sel):
            if v[i] == capi.CEC_NOT_EQUIVALENT:
                po_v[q] = capi.CEC_NOT_EQUIVALENT
            elif v[i] == capi.CEC_EQUIVALENT:
                po_v[q] = capi.CEC_EQUIVALENT
        neq = [int(q) for i, q in enumerate(sel) if v[i] == capi.CEC_NOT_EQUIVALENT]
        if neq:
            q0 = min(neq)
            i0 = int(np.nonzero(sel == q0)[0][0])
            vec = ctx.get_cex(i0)
            log.append({"phase": "P", "threshold": thr, "simulated": int(sel.size), "neq": len(neq),
                        "s": time.perf_counter() - t})
            return CecResult(capi.CEC_NOT_EQUIVALENT, po_v, cex=vec, cex_pair=q0, log=log, final_ands=cur.aig.num_ands)
        for i, q in enumerate(sel):
            if v[i] == capi.CEC_EQUIVALENT:
                a, b = int(cur.lit_a[q]), int(cur.lit_b[q])
                hi, lo = (a, b) if (a >> 1) > (b >> 1) else (b, a)
                # an identical node pair (a >> 1 == b >> 1) needs no merge (and merging a node
                # into itself is not a reduction)
                if (hi >> 1) > cur.aig.num_pis and (hi >> 1) != (lo >> 1):
                    subst[hi >> 1] = lo ^ (hi & 1)
    log.append({"phase": "P", "threshold": thr, "simulated": int(sel.size), "s": time.perf_counter() - t})
    if subst:
        cur, _ = cur.reduce(subst, p.device, ctx=ctx)

    # ---- G and L phases -----------------------------------------------------------------------
    tried_global = set()
    cex_patterns: List[np.ndarray] = []  # CEXs of refuted candidate pairs (class refinement)
    for phase_no in range(p.max_phases):
        st = po_status(cur)
        if (st == capi.CEC_EQUIVALENT).all():
            break
        t = time.perf_counter()
        # local checks need k_max >= k_l (cut leaves); one context serves both when k_l <= k_g
        ctx = dctx(cur, p.k_g)
        lctx = ctx if p.k_l <= p.k_g else dctx(cur, max(p.k_l, 1), slot=1)
        t_ctx = time.perf_counter() - t
        # equivalence classes on the GPU: random patterns plus the CEX patterns
        # of disproved pairs, which split their classes
        words = pack_patterns(cex_patterns, cur.aig.num_pis) if cex_patterns else None
        tk = {"ctx": t_ctx, "classes": 0.0, "global": 0.0, "cuts": 0.0, "local": 0.0}
        t1 = time.perf_counter()
        cr, cm, cf = ctx.sim_classes(p.sim_words, p.seed + phase_no, words)
        tk["classes"] += time.perf_counter() - t1
        cand = [(int(r), int(m_), int(f)) for r, m_, f in zip(cr, cm, cf)]
        versions.append(cur.aig)
        # G phase once per miter version: pairs with support <= k_g
        gl = [(r, m_, f) for r, m_, f in cand if (r, m_, f) not in tried_global]
        la = [2 * r for r, m_, f in gl]
        lb = [2 * m_ ^ f for r, m_, f in gl]
        subst = {}
        proved_g = 0
        if gl:
            t1 = time.perf_counter()
            v, _, k = ctx.sim_exhaustive(la, lb)
            tk["global"] += time.perf_counter() - t1
            for i in np.nonzero(v == capi.CEC_NOT_EQUIVALENT)[0][:p.max_cex_patterns]:
                if len(cex_patterns) >= p.max_cex_patterns:
                    break
                cx = ctx.get_cex(int(i))
                cex_patterns.append(cx)
                if p.distance1:  # distance-1 simulation of the CEX over the pair's support
                    for pi in capi.cec_pair_support(ctx.handle, la[i], lb[i]):
                        if len(cex_patterns) >= p.max_cex_patterns:
                            break
                        nb = cx.copy()
                        nb[pi - 1] ^= 1
                        cex_patterns.append(nb)
            for (r, m_, f), vv in zip(gl, v):
                if vv == capi.CEC_EQUIVALENT and m_ not in subst:
                    subst[m_] = 2 * r ^ f
                    proved_g += 1
                if vv != capi.CEC_UNDECIDED:
                    tried_global.add((r, m_, f))
        remaining = [(r, m_, f) for r, m_, f in cand if m_ not in subst and (r, m_, f) not in tried_global]
        # L: 3 passes of cut enumeration + local checks (Table I)
        proved_l = 0
        for pass_id in range(3):
            if not remaining:
                break
            todo = [x for x in remaining if x[1] not in subst]
            ql, qm, off, leaves, who = [], [], [0], [], []
            if p.native_cuts and todo:
                # Alg. 2: level-wise cut enumeration, common-cut buffer flushed
                # to the local-check kernels while the host enumerates the next levels
                t1 = time.perf_counter()
                pv, (cp, cof, cl, cv) = capi.cec_local_pass(
                    lctx.handle, [x[0] for x in todo], [x[1] for x in todo], [x[2] for x in todo], p.k_l, p.C,
                    pass_id, p.max_cuts_per_pair, p.buffer_checks)
                tk["local"] += time.perf_counter() - t1
                ver = len(versions) - 1
                if cp.size:
                    ta = np.array([x[0] for x in todo], dtype=np.int64)
                    tm_ = np.array([x[1] for x in todo], dtype=np.int64)
                    tf = np.array([x[2] for x in todo], dtype=np.int64)
                    idx = cp.astype(np.int64)
                    checks.add(ver, phase_no, pass_id, 2 * ta[idx], (2 * tm_[idx]) ^ tf[idx], cof, cl, cv)
                for i, (r, m_, f) in enumerate(todo):
                    if pv[i] == capi.CEC_EQUIVALENT and m_ not in subst:
                        subst[m_] = 2 * r ^ f
                        proved_l += 1
                remaining = [x for x in remaining if x[1] not in subst]
                continue
            elif todo:
                repr_of = {m_: r for r, m_, f in todo}
                cuts = enumerate_cuts(cur.aig, p.k_l, p.C, pass_id, repr_of)
                for r, m_, f in todo:
                    common = set()
                    for u in cuts[r]:
                        for v_ in cuts[m_]:
                            c = u | v_
                            if c.bit_count() <= p.k_l:
                                common.add(c)
                    for c in sorted(common, key=lambda x: (x.bit_count(), x))[:p.max_cuts_per_pair]:
                        ql.append(2 * r)
                        qm.append(2 * m_ ^ f)
                        leaves += _bits(c)
                        off.append(len(leaves))
                        who.append((r, m_, f))
            if not ql:
                continue
            t1 = time.perf_counter()
            lv = lctx.check_local_cuts(ql, qm, off, leaves)
            tk["local"] += time.perf_counter() - t1
            for q, vv in enumerate(lv):
                checks.append({"version": len(versions) - 1, "phase": phase_no, "pass": pass_id,
                               "lit_a": ql[q], "lit_b": qm[q], "leaves": leaves[off[q]:off[q + 1]], "verdict": int(vv)})
                r, m_, f = who[q]
                if vv == capi.CEC_EQUIVALENT and m_ not in subst:
                    subst[m_] = 2 * r ^ f
                    proved_l += 1
            remaining = [x for x in remaining if x[1] not in subst]
        entry = {"phase": f"G+L{phase_no}", "candidates": len(cand), "proved_global": proved_g,
                 "proved_local": proved_l, "ands": cur.aig.num_ands,
                 "s_parts": {k_: round(v_, 4) for k_, v_ in tk.items()}}
        log.append(entry)
        if subst:
            t1 = time.perf_counter()
            nxt, image = cur.reduce(subst, p.device, ctx=ctx)
            entry["s_parts"]["reduce"] = round(time.perf_counter() - t1, 4)
        entry["s"] = time.perf_counter() - t
        if not subst:
            break  # no progress: undecided remainder
        cur = nxt
        # tried_global holds node ids of the old version: carry each decided pair over to its image
        # in the new one (the reduction preserves every node's function), so a refuted pair is not
        # re-simulated and a new pair that reuses old ids is not skipped
        tried_global = _remap_tried(tried_global, image)
    st = po_status(cur)
    po_v = np.where(st == capi.CEC_EQUIVALENT, capi.CEC_EQUIVALENT, po_v)
    cex_vec, cex_pair = None, -1
    if p.final_po_check and (po_v != capi.CEC_EQUIVALENT).any():
        # The P phase only simulated POs with k <= k_p when some PO exceeded k_P.
        # On the reduced miter, the still-undecided POs with k <= k_P are decided exhaustively
        # (an extension of the paper's flow, which hands them to ABC instead).
        t = time.perf_counter()
        hctx = capi.Context.from_aig(cur.aig, device=-1, k_max=63)
        und = [q for q in range(P) if po_v[q] != capi.CEC_EQUIVALENT and
               hctx.pair_k(int(cur.lit_a[q]), int(cur.lit_b[q])) <= p.k_P]
        hctx.close()
        if und:
            ctx = dctx(cur, p.k_P)
            v, _, _ = ctx.sim_exhaustive(cur.lit_a[und], cur.lit_b[und])
            for i, q in enumerate(und):
                if v[i] != capi.CEC_UNDECIDED:
                    po_v[q] = v[i]
            neq = [i for i, q in enumerate(und) if v[i] == capi.CEC_NOT_EQUIVALENT]
            if neq:
                cex_vec, cex_pair = ctx.get_cex(neq[0]), und[neq[0]]
        log.append({"phase": "final-P", "threshold": p.k_P, "simulated": len(und), "s": time.perf_counter() - t})
    if (po_v == capi.CEC_NOT_EQUIVALENT).any():
        verdict = capi.CEC_NOT_EQUIVALENT
    elif (po_v == capi.CEC_EQUIVALENT).all():
        verdict = capi.CEC_EQUIVALENT
    else:
        verdict = capi.CEC_UNDECIDED
    return CecResult(verdict, po_v, cex=cex_vec, cex_pair=cex_pair, log=log, checks=checks, versions=versions,
                     final_ands=cur.aig.num_ands)
