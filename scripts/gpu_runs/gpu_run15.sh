set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1"
timeout 600 $B --config c2 > gpurun_out/p_c2.log 2>&1
timeout 900 $B > gpurun_out/p_c5.log 2>&1
timeout 900 $B --config c3 > gpurun_out/p_c3.log 2>&1
timeout 2000 python -m pytest tests/test_gpu_parity.py -m gpu -q -rf -x -k "fuzz or c2_full or c5_reduced or small_mult or c5_full" > gpurun_out/pytest_gpu.log 2>&1
echo done
