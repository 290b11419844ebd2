"""compute-sanitizer memcheck / racecheck / synccheck over both engines on small miters
(SURVEY.md §4.2 "Sanitizers"). Runs the check in a subprocess under the sanitizer."""
import os
import shutil
import subprocess
import sys

import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SCRIPT = r"""
import sys
sys.path.insert(0, %r)
from paper_conf_dac_liuy25_b200 import capi
from workloads import c1_add8, circuits
# JIT: c1 / mul6 run as single-structure free-warp kernels with IMAD cells; the reduced C5 as a
# block-synchronous bundle kernel (several structures)
mini = circuits.c5_big(copies=4, n_random=2, n_bugs=1, rand_pis=12, rand_ands=200, mul_n=6)
for eng in (capi.CEC_ENGINE_INTERP, capi.CEC_ENGINE_JIT):
    for m in (c1_add8(), circuits.c2_mul12_bug(seed=1, n=6), mini):
        ctx = capi.Context.from_aig(m.aig, engine=eng)
        v, c, k = ctx.sim_exhaustive(m.lit_a, m.lit_b)
        ctx.check_local_cuts(m.lit_a[:2], m.lit_b[:2], [0, 2, 4], [1, 2, 3, 4])
        capi.cec_sim_random(ctx.handle, m.aig.num_nodes, 8, 1)
        ctx.close()
print("SANITIZER-RUN-OK")
""" % ROOT


@pytest.mark.parametrize("tool", ["memcheck", "racecheck", "synccheck"])
def test_compute_sanitizer(tool):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    # opt-in: on the B200 pool, runs under compute-sanitizer have left GPUs needing a reset (the
    # operators disabled the tool there); the round-2 runs with 0 errors are in profiles/
    if os.environ.get("CEC_RUN_SANITIZER") != "1":
        pytest.skip("compute-sanitizer runs are opt-in (CEC_RUN_SANITIZER=1)")
    cs = shutil.which("compute-sanitizer") or "/usr/local/cuda/bin/compute-sanitizer"
    if not os.path.exists(cs):
        pytest.skip("compute-sanitizer not found")
    r = subprocess.run([cs, "--tool", tool, "--error-exitcode", "9", sys.executable, "-c", SCRIPT],
                       capture_output=True, text=True, timeout=1200)
    if "closed on this pool" in r.stdout + r.stderr:  # the GPU pool's operators disabled the tool
        pytest.skip("compute-sanitizer is disabled on this GPU pool: " + (r.stdout + r.stderr).strip()[:200])
    assert "SANITIZER-RUN-OK" in r.stdout, r.stdout[-2000:] + r.stderr[-2000:]
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-2000:]
    out = r.stdout + r.stderr
    assert "ERROR SUMMARY: 0 errors" in out or "RACECHECK SUMMARY: 0 hazards displayed (0 errors, 0 warnings)" in out, out
