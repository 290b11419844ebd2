set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
B="python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1"
timeout 300 $B > gpurun_out/t_default.log 2>&1
CEC_JIT_SYNC=0 CEC_JIT_THREADS=128 CEC_JIT_MINB=4 timeout 300 $B > gpurun_out/t_warp128.log 2>&1
CEC_JIT_SYNC=128 timeout 300 $B > gpurun_out/t_sync128.log 2>&1
CEC_JIT_SYNC=512 timeout 300 $B > gpurun_out/t_sync512.log 2>&1
CEC_JIT_SYNC=64 timeout 300 $B > gpurun_out/t_sync64.log 2>&1
CEC_JIT_THREADS=256 CEC_JIT_MINB=2 timeout 300 $B > gpurun_out/t_256x2.log 2>&1
timeout 300 $B --config c2 > gpurun_out/t_c2.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -rf -x > gpurun_out/pytest_gpu.log 2>&1
echo done
