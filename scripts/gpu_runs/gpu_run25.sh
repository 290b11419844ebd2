mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests -q -m gpu -x -k "supports or pipelined or c5 or driver" > gpurun_out/test_gpu.log 2>&1
timeout 600 python scripts/time_plan.py c5 4 > gpurun_out/timing.log 2>&1
for K in 4 6 8 12; do CEC_PIPELINE=$K timeout 600 python scripts/time_plan.py c5 3 2>&1 | grep "^---" | tail -1 | sed "s/^/K=$K /" >> gpurun_out/timing_k.log; done
echo done
