set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 1800 python -m pytest tests/test_gpu_parity.py -m gpu -q -rf -x -k "fuzz or c1 or small_mult or invariance or c5_reduced or c2_full" > gpurun_out/pytest_simt.log 2>&1
B="python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1"
timeout 900 $B --engine 3 > gpurun_out/s_c5.log 2>&1
timeout 600 $B --engine 3 --config c2 > gpurun_out/s_c2.log 2>&1
echo done
