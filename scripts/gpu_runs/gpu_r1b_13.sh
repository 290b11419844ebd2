mkdir -p gpurun_out/t13
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/t13/build.log 2>&1
timeout 600 python scripts/time_plan.py c3 4 > gpurun_out/t13/c3_timing.log 2>&1
timeout 600 python scripts/time_plan.py c5 4 > gpurun_out/t13/c5_timing.log 2>&1
nproc > gpurun_out/t13/nproc.txt; lscpu | head -20 > gpurun_out/t13/lscpu.txt
echo done
