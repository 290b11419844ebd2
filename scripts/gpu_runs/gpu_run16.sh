set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1"
timeout 900 $B > gpurun_out/sp_c5.log 2>&1
CEC_JIT_SPLICE=0 timeout 900 $B > gpurun_out/sp_c5_off.log 2>&1
timeout 900 $B --config c3 > gpurun_out/sp_c3.log 2>&1
timeout 600 $B --config c2 > gpurun_out/sp_c2.log 2>&1
timeout 3000 python -m pytest tests -m gpu -q -rf > gpurun_out/pytest_gpu.log 2>&1
echo done
