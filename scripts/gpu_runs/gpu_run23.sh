mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -q -m gpu -x -k "supports or c5 or rerun or invariance" > gpurun_out/test_gpu.log 2>&1
timeout 600 python scripts/time_plan.py c5 4 > gpurun_out/timing.log 2>&1
timeout 900 python bench.py > gpurun_out/bench_c5.log 2>&1
echo done
