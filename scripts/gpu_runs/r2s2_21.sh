# round 2 (re-entry): full GPU suite on the current tree; C5 public-call tail phases
set -x
mkdir -p gpurun_out/r2s2_21
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r2s2_21/smoke.log 2>&1
timeout 300 python scripts/time_plan.py c5 3 > gpurun_out/r2s2_21/c5.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -rf > gpurun_out/r2s2_21/pytest_gpu.log 2>&1
echo done
