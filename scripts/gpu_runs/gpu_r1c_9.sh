# round 1c: regression after the support-table cache; e2e timing
mkdir -p gpurun_out/c9
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c9/build.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu -rf -x > gpurun_out/c9/pytest.log 2>&1
CEC_TIMING=1 timeout 300 python scripts/time_plan.py c5 3 > gpurun_out/c9/time_plan.log 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/c9/bench.log 2>&1
timeout 600 python bench.py --no-cpu-baseline --config c3 > gpurun_out/c9/bench_c3.log 2>&1
echo done
