# round 2, run 18: free-warp bundles (C3) A/B vs single-only (CEC_JIT_FREE=1) and block-sync (0); full GPU suite
set -x
mkdir -p gpurun_out/r2_18
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r2_18/smoke.log 2>&1
B="python bench.py --steps 20 --warmup 5 --no-cpu-baseline --e2e-steps 3"
timeout 600 $B --config c3 > gpurun_out/r2_18/c3_free2.log 2>&1
CEC_JIT_FREE=1 timeout 600 $B --config c3 > gpurun_out/r2_18/c3_free1.log 2>&1
CEC_JIT_FREE=0 timeout 600 $B --config c3 > gpurun_out/r2_18/c3_free0.log 2>&1
timeout 600 $B > gpurun_out/r2_18/c5_free2.log 2>&1
timeout 300 $B --config c2 > gpurun_out/r2_18/c2_free2.log 2>&1
timeout 300 $B --config c1 > gpurun_out/r2_18/c1_free2.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -rf -x > gpurun_out/r2_18/pytest_gpu.log 2>&1
echo done
