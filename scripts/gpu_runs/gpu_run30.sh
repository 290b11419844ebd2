mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
CEC_TIMING=1 timeout 900 python bench.py --config c3 --no-cpu-baseline --steps 3 --e2e-steps 3 > gpurun_out/bench_c3_t.log 2>&1
CEC_PIPELINE=1 CEC_TIMING=1 timeout 900 python bench.py --config c3 --no-cpu-baseline --steps 3 --e2e-steps 3 > gpurun_out/bench_c3_t1.log 2>&1
echo done
