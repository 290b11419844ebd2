"""Command line of the GPU path with the oracle CLI's diffable output (SURVEY.md §8(c) "Diffable
output"): the same files in, byte-identical text out when the two agree.

  python -m paper_conf_dac_liuy25_b200.cli check <aag> <pairs> [k_max]
  python -m paper_conf_dac_liuy25_b200.cli local <aag> <checks>

check: one line per pair `pair_idx lit_a lit_b k EQ|NEQ|UND cex_index|-`, then for every NEQ pair
`cex pair_idx <hex of the PI values, PI 1 = bit 0>` (cec_sim_exhaustive + cec_get_cex on cuda:0).
local: one line per check `check_idx lit_a lit_b leaves... EQ|UND` (cec_check_local_cuts).
Files: pairs = `n` then n lines `lit_a lit_b`; checks = `n` then n lines `lit_a lit_b m leaf_1..leaf_m`
(workloads.write_pairs / write_checks)."""
import sys

import numpy as np

from . import capi
from workloads.aig import read_aag

NAMES = {capi.CEC_EQUIVALENT: "EQ", capi.CEC_NOT_EQUIVALENT: "NEQ", capi.CEC_UNDECIDED: "UND"}


def _hex_bits(bits) -> str:
    n = len(bits)
    nib = (n + 3) // 4
    if nib == 0:
        return "0"
    out = []
    for h in range(nib - 1, -1, -1):
        v = 0
        for b in range(3, -1, -1):
            i = h * 4 + b
            v = (v << 1) | (int(bits[i]) if i < n else 0)
        out.append("%x" % v)
    return "".join(out)


def _ints(path):
    with open(path) as fh:
        return [int(x) for x in fh.read().split()]


def main(argv=None) -> int:
    argv = sys.argv[1:] if argv is None else argv
    if len(argv) < 3 or argv[0] not in ("check", "local"):
        print(__doc__, file=sys.stderr)
        return 2
    aig = read_aag(argv[1])
    t = _ints(argv[2])
    n, out = t[0], []
    if argv[0] == "check":
        k_max = int(argv[3]) if len(argv) > 3 else 32
        la = np.array(t[1:1 + 2 * n:2], dtype=np.uint32)
        lb = np.array(t[2:2 + 2 * n:2], dtype=np.uint32)
        ctx = capi.Context.from_aig(aig, device=0, k_max=k_max)
        v, cex, k = ctx.sim_exhaustive(la, lb)
        for p in range(n):
            tail = str(int(cex[p])) if v[p] == capi.CEC_NOT_EQUIVALENT else "-"
            out.append(f"{p} {int(la[p])} {int(lb[p])} {int(k[p])} {NAMES[int(v[p])]} {tail}")
        for p in range(n):
            if v[p] == capi.CEC_NOT_EQUIVALENT:
                out.append(f"cex {p} {_hex_bits(ctx.get_cex(p))}")
    else:
        la, lb, off, lv, pos = [], [], [0], [], 1
        for _ in range(n):
            a, b, m = t[pos], t[pos + 1], t[pos + 2]
            la.append(a)
            lb.append(b)
            lv += t[pos + 3:pos + 3 + m]
            off.append(len(lv))
            pos += 3 + m
        ctx = capi.Context.from_aig(aig, device=0, k_max=max(1, max((off[i + 1] - off[i] for i in range(n)), default=1)))
        v = ctx.check_local_cuts(la, lb, off, lv)
        for q in range(n):
            leaves = " ".join(str(x) for x in lv[off[q]:off[q + 1]])
            out.append(f"{q} {la[q]} {lb[q]}" + (f" {leaves}" if leaves else "") + f" {NAMES[int(v[q])]}")
    ctx.close()
    sys.stdout.write("\n".join(out) + ("\n" if out else ""))
    return 0


if __name__ == "__main__":
    sys.exit(main())
