# round 2 (re-entry): C4 flow with one reloaded device context (cec_reload_aig), spinning worker
# pool, parallel small cut levels; driver/local GPU tests; C3/C5 public-call timing (no regression)
set -x
mkdir -p gpurun_out/r2s2_11
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2s2_11/build.log 2>&1
CEC_TIMING_LOCAL=1 timeout 600 python scripts/c4_flow.py > gpurun_out/r2s2_11/c4.log 2> gpurun_out/r2s2_11/c4.err
timeout 1500 python -m pytest tests/test_gpu_local_pass.py tests/test_gpu_parity.py tests/test_gpu_classes.py tests/test_gpu_reduce.py -q -rf -k "local or cut or c4 or driver or classes or reduce" > gpurun_out/r2s2_11/pytest.log 2>&1
timeout 300 python scripts/time_plan.py c3 4 > gpurun_out/r2s2_11/c3.log 2>&1
timeout 300 python scripts/time_plan.py c5 3 > gpurun_out/r2s2_11/c5.log 2>&1
echo done
