# round 2 (re-entry): C3 host planning (no zero fill of programs; id order skipped for small interpreter
# windows): timing + full GPU suite
set -x
mkdir -p gpurun_out/r2s2_16
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r2s2_16/smoke.log 2>&1
timeout 300 python scripts/time_plan.py c3 5 > gpurun_out/r2s2_16/c3.log 2>&1
timeout 600 python bench.py --steps 20 --warmup 5 --config c3 --no-cpu-baseline > gpurun_out/r2s2_16/bench_c3.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -rf > gpurun_out/r2s2_16/pytest_gpu.log 2>&1
echo done
