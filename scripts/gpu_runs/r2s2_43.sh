# round 2 (re-entry): GPU cone sizes for C3's cost-aware merge: test vs host walk, C3 call timing, bench
set -x
mkdir -p gpurun_out/r2s2_43
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2s2_43/build.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -rf -k "cone_sizes or c3_full or split or bundles" > gpurun_out/r2s2_43/pytest.log 2>&1
timeout 300 python scripts/time_plan.py c3 5 > gpurun_out/r2s2_43/c3.log 2>&1
CEC_CONES_GPU=0 timeout 300 python scripts/time_plan.py c3 5 > gpurun_out/r2s2_43/c3_host.log 2>&1
timeout 600 python bench.py --steps 20 --warmup 5 --config c3 --no-cpu-baseline > gpurun_out/r2s2_43/bench_c3.log 2>&1
echo done
