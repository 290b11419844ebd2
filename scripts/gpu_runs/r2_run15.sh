# round 2, run 15: free-warp kernels (default for single small structures) vs block-synchronous (CEC_JIT_FREE=0)
set -x
mkdir -p gpurun_out/r2_15
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r2_15/smoke.log 2>&1
B="python bench.py --steps 20 --warmup 5 --no-cpu-baseline --e2e-steps 3"
timeout 300 $B --config c2 > gpurun_out/r2_15/c2_free.log 2>&1
CEC_JIT_FREE=0 timeout 300 $B --config c2 > gpurun_out/r2_15/c2_sync.log 2>&1
timeout 300 $B --config c2bug > gpurun_out/r2_15/c2bug_free.log 2>&1
timeout 600 $B > gpurun_out/r2_15/c5_free.log 2>&1
CEC_JIT_FREE=0 timeout 600 $B > gpurun_out/r2_15/c5_sync.log 2>&1
timeout 600 $B --config c3 > gpurun_out/r2_15/c3_free.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -rf -x > gpurun_out/r2_15/pytest_gpu.log 2>&1
echo done
