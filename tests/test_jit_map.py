"""CPU tests of the JIT window compiler's cell mapping (csrc/jit.cpp), host only (NVRTC/nvJitLink
run without a GPU; nothing is launched).

The kernels evaluate each window as a network of cells: 3-input LUTs (one lop3.b32 each, ALU pipe)
and, in mapping mode 3, IMAD cells (one mad.lo.u32 each, FMA pipe) for AND nodes with a
word-uniform window input m (input index >= 5: every u32 word of it is 0 or ~0), using
y*m + m = ~y & m, y*m + y = y & ~m and y*m - 1 = ~(y & m). CEC_JIT_VERIFY=1 makes the compiler
evaluate every mapped network exactly as the body executes it (LOP3 tables over stored values,
32-bit wrap-around mads, register polarities) on random word-uniform input words and compare
every cell and every compare's diff with the AIG's own AND evaluation; a mismatch fails the plan.
Each check runs in a fresh process so the process-wide kernel cache cannot skip the verification."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

SCRIPT = r"""
import json, sys
sys.path.insert(0, {root!r})
from paper_conf_dac_liuy25_b200 import capi
from workloads import circuits
name = {name!r}
if name == "c2":
    m = circuits.c2_mul12()
elif name == "mul8bug":
    m = circuits.c2_mul12_bug(seed=1, n=8)
elif name == "c5mini":
    m = circuits.c5_big(copies=6, n_random=4, n_bugs=2, rand_pis=16, rand_ands=900, mul_n=8)
elif name.startswith("rand"):
    s = int(name[4:])
    m = circuits.random_miter(14 + s % 6, 300 + 40 * s, 8, seed=100 + s, window=24 + s)
ctx = capi.Context.from_aig(m.aig, device=-1, engine=capi.CEC_ENGINE_JIT, merge={merge})
plan = capi.cec_plan_exhaustive(ctx.handle, m.lit_a, m.lit_b)
st = ctx.stats()
W = capi.cec_plan_info(plan)["node_patterns"]
capi.cec_plan_free(plan)
print(json.dumps({{"lop3": st["lop3_words"], "imad": st["imad_words"], "W": W, "jit": st["jit_windows"]}}))
"""


def plan_stats(name, mode, verify=True, merge=1):
    env = dict(os.environ, CEC_JIT_FUSE=str(mode))
    if verify:
        env["CEC_JIT_VERIFY"] = "1"
    r = subprocess.run([sys.executable, "-c", SCRIPT.format(root=ROOT, name=name, merge=merge)], env=env,
                       capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    return json.loads(r.stdout.strip().splitlines()[-1])


@pytest.mark.parametrize("name", ["c2", "mul8bug", "c5mini", "rand0", "rand1", "rand2", "rand3", "rand4", "rand5"])
def test_mapped_networks_equal_the_aig(name):
    """Both mappings (mode 2: LUTs only; mode 3: LUTs + IMAD cells) pass the host emulation check on
    every window structure, and mode 3 moves work off the LOP3 pipe: fewer LUT words, some IMADs."""
    s2 = plan_stats(name, 2)
    s3 = plan_stats(name, 3)
    assert s2["jit"] >= 1 and s2["imad"] == 0 and s2["W"] == s3["W"]
    assert s3["lop3"] <= s2["lop3"]
    if name in ("c2", "c5mini"):
        assert s3["imad"] > 0 and s3["lop3"] < s2["lop3"]


def test_verifier_detects_a_wrong_cell(tmp_path):
    """The emulation check is live: a window whose IMAD forms are deliberately broken
    (CEC_JIT_BREAK_IMAD, test hook) fails the plan with the mismatching cell named."""
    env = dict(os.environ, CEC_JIT_FUSE="3", CEC_JIT_VERIFY="1", CEC_JIT_BREAK_IMAD="1")
    r = subprocess.run([sys.executable, "-c", SCRIPT.format(root=ROOT, name="c2", merge=1)], env=env,
                       capture_output=True, text=True, timeout=600)
    assert r.returncode != 0 and "mapped cell of node" in r.stderr
