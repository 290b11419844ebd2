# JIT bundles: full GPU suite, C3/C5/C2 bench
mkdir -p gpurun_out/t6
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/t6/smoke.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu -rf -x > gpurun_out/t6/pytest_gpu.log 2>&1
timeout 900 python bench.py --config c3 --no-cpu-baseline > gpurun_out/t6/c3.log 2>&1
CEC_PROFILE_GROUPS=1 timeout 600 python scripts/profile_groups.py c3 > gpurun_out/t6/c3_groups.log 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/t6/c5.log 2>&1
timeout 300 python bench.py --config c2 --no-cpu-baseline > gpurun_out/t6/c2.log 2>&1
echo done
