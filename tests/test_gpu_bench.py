"""GPU test of bench.py's own arm (task contract ④): ONE JSON line with every contract key, the
roofline object (bound / achieved / peak / unit / frac / traffic and the window-kernel time), the
clocks sampled during the timed region, the end-to-end object with its copy bytes, the launch count,
the SURVEY.md §8(d) record, and parity 0 diffs against the stored oracle results."""
import json
import os
import subprocess
import sys

import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_bench_gpu_arm_json_line():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--config", "c1", "--steps", "3",
                        "--warmup", "3", "--no-cpu-baseline"], capture_output=True, text=True, timeout=900, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    for key in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
                "vs_baseline", "dtype", "data", "config", "clocks", "e2e", "gpu_launches", "roofline", "record",
                "parity"):
        assert key in d, key
    assert d["n_gpus"] == 1 and d["steps"] == 3 and d["warmup"] >= 3 and d["value"] > 0
    assert d["config"]["workload"] == "c1" and d["dtype"] == "u32" and d["gpu_launches"] > 0
    ro = d["roofline"]
    for key in ("bound", "achieved", "peak", "unit", "frac", "traffic", "kernel_ms", "step_frac"):
        assert key in ro, key
    assert ro["bound"] == "alu" and 0 < ro["frac"] <= 1.0 and ro["kernel_ms"] > 0
    e = d["e2e"]
    assert e["value"] > 0 and e["h2d_bytes_per_step"] > 0 and e["d2h_bytes_per_step"] > 0
    assert "sm_mhz" in d["clocks"] and "reasons" in d["clocks"]
    assert d["parity"]["ok"] and d["parity"]["diffs"] == 0
    rec = d["record"]
    for key in ("config", "seed", "gpus", "W", "t_kernel_ms", "node_patterns_per_s", "t_e2e_ms", "t_hostprep_ms",
                "t_h2d_ms", "t_allreduce_us", "dram_GBps", "alu_pipe_pct", "lop3_count_per_W32", "sm_clock_MHz",
                "oracle_wall_s", "oracle_cores", "oracle_cpu_s", "parity"):
        assert key in rec, key
