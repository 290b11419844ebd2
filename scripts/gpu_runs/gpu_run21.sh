mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
nproc > gpurun_out/timing.log; lscpu | grep -i "model name\|^CPU(s)\|Thread\|MHz" >> gpurun_out/timing.log
timeout 600 python scripts/time_plan.py c5 4 >> gpurun_out/timing.log 2>&1
timeout 600 python scripts/time_plan.py c3 3 >> gpurun_out/timing.log 2>&1
timeout 600 python scripts/time_plan.py c2 3 >> gpurun_out/timing.log 2>&1
echo done
