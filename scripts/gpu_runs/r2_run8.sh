# round 2, run 8: host phase timings (CEC_TIMING) of the e2e call for C3 and C5
set -x
mkdir -p gpurun_out/r2_8
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2_8/build.log 2>&1
nproc > gpurun_out/r2_8/nproc.txt; lscpu | head -20 >> gpurun_out/r2_8/nproc.txt
CEC_TIMING=1 timeout 600 python bench.py --config c3 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 3 > gpurun_out/r2_8/timing_c3.log 2>&1
CEC_TIMING=1 timeout 600 python bench.py --config c5 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 3 > gpurun_out/r2_8/timing_c5.log 2>&1
echo done
