set -x
mkdir -p gpurun_out
nproc > gpurun_out/nproc.txt; lscpu | head -20 >> gpurun_out/nproc.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
CEC_TIMING=1 timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 3 > gpurun_out/t_c5.log 2> gpurun_out/t_c5.err
timeout 3000 python -m pytest tests -m gpu -q -rf > gpurun_out/pytest_gpu.log 2>&1
echo done
