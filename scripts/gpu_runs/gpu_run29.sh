mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu -x > gpurun_out/test_gpu.log 2>&1
timeout 600 python scripts/time_plan.py c5 3 > gpurun_out/timing.log 2>&1
timeout 900 python bench.py > gpurun_out/bench_c5.log 2>&1
timeout 900 python bench.py --config c3 --no-cpu-baseline > gpurun_out/bench_c3.log 2>&1
timeout 900 python bench.py --config c2 --no-cpu-baseline > gpurun_out/bench_c2.log 2>&1
echo done
