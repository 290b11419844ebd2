mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 python -m pytest tests -q -m gpu -x -k "supports or pipelined or c5_full" > gpurun_out/test_gpu.log 2>&1
timeout 600 python scripts/time_plan.py c5 4 > gpurun_out/timing.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:supp --csv --log-file gpurun_out/supp_launches.csv python scripts/time_plan.py c5 2 > /dev/null 2>&1
echo done
