"""Run the CEC driver (P/G/L flow) on C4 and its bug variant; print the phase log as JSON lines.

SURVEY.md §8(d)(ii): CUDA context creation and JIT compiles are excluded from the end-to-end time
and reported once, so one untimed warm-up of each flow (C4, C4-bug) runs first (its wall time is printed as
`warmup_seconds` on the first line)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_dac_liuy25_b200 import capi, driver  # noqa: E402
from workloads import c4_dp  # noqa: E402

t0 = time.perf_counter()
for m0 in (c4_dp(64), c4_dp(64, bug=4)):  # both flows once: the bug flow's final PO check JIT-compiles
    driver.check_miter(m0.aig, m0.lit_a, m0.lit_b, driver.CecParams(k_l=16, C=16))
warm = round(time.perf_counter() - t0, 2)
for name, m in (("c4_dp64", c4_dp(64)), ("c4_dp64_bug4", c4_dp(64, bug=4))):
    t = time.perf_counter()
    r = driver.check_miter(m.aig, m.lit_a, m.lit_b, driver.CecParams(k_l=16, C=16))
    dt = time.perf_counter() - t
    names = {capi.CEC_EQUIVALENT: "EQ", capi.CEC_NOT_EQUIVALENT: "NEQ", capi.CEC_UNDECIDED: "UND"}
    print(json.dumps({"miter": name, "verdict": names[r.verdict], "seconds": round(dt, 2), "warmup_seconds": warm,
                      "po_eq": int((r.po_verdicts == capi.CEC_EQUIVALENT).sum()),
                      "po_neq": int((r.po_verdicts == capi.CEC_NOT_EQUIVALENT).sum()),
                      "po_und": int((r.po_verdicts == capi.CEC_UNDECIDED).sum()),
                      "local_checks": len(r.checks), "final_ands": r.final_ands, "start_ands": int(m.aig.num_ands),
                      "log": r.log}), flush=True)
