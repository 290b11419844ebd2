# round 2 (re-entry): C3 engine-aware split pipelining A/B (CEC_PIPE_SPLIT=0 = old single chunk)
set -x
mkdir -p gpurun_out/r2s2_2
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2s2_2/build.log 2>&1
CEC_PIPE_SPLIT=0 timeout 600 python scripts/time_plan.py c3 4 > gpurun_out/r2s2_2/time_plan_c3_off.log 2>&1
timeout 600 python scripts/time_plan.py c3 4 > gpurun_out/r2s2_2/time_plan_c3_split.log 2>&1
timeout 600 python bench.py --steps 20 --warmup 5 --config c3 --no-cpu-baseline > gpurun_out/r2s2_2/bench_c3.log 2>&1
CEC_PIPE_SPLIT=0 timeout 600 python bench.py --steps 20 --warmup 5 --config c3 --no-cpu-baseline > gpurun_out/r2s2_2/bench_c3_off.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "c3 or split or pipelined or bundles" > gpurun_out/r2s2_2/pytest_c3.log 2>&1
echo done
