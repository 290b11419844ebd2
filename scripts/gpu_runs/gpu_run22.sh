mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 python scripts/time_plan.py c5 4 > gpurun_out/timing.log 2>&1
timeout 600 python scripts/time_plan.py c3 4 >> gpurun_out/timing.log 2>&1
timeout 600 python scripts/time_plan.py c2 4 >> gpurun_out/timing.log 2>&1
timeout 1200 python -m pytest tests -q -m gpu -x > gpurun_out/test_gpu.log 2>&1
echo done
