set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
B="python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 --config c3"
timeout 900 $B > gpurun_out/c3_26.log 2>&1
CEC_JIT_MIN_NODE_WORDS=8388608 timeout 900 $B > gpurun_out/c3_23.log 2>&1
CEC_JIT_MIN_NODE_WORDS=1048576 timeout 900 $B > gpurun_out/c3_20.log 2>&1
timeout 900 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 --config c3 --engine 1 > gpurun_out/c3_interp.log 2>&1
timeout 3000 python -m pytest tests -m gpu -q -rf -k "sanitizer or nccl or sim_patterns or driver" > gpurun_out/pytest_gpu.log 2>&1
echo done
