# round 2, run 12: pipelined e2e call without side-stream joins between chunks (A/B), pipeline tests
set -x
mkdir -p gpurun_out/r2_12
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2_12/build.log 2>&1
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 7"
timeout 600 $B > gpurun_out/r2_12/nojoin.log 2>&1
CEC_PIPE_JOIN=1 timeout 600 $B > gpurun_out/r2_12/join.log 2>&1
timeout 600 $B > gpurun_out/r2_12/nojoin2.log 2>&1
CEC_PIPE_JOIN=1 timeout 600 $B > gpurun_out/r2_12/join2.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -rf -x -k "pipelined or c5_full or jit_bundles" > gpurun_out/r2_12/pytest.log 2>&1
echo done
