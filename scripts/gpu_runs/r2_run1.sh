# round 2, run 1: verify the ADVICE fixes on a fresh B200 (GPU tests, smoke, default bench, c3/c2)
set -x
mkdir -p gpurun_out/r2_1
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r2_1/smoke.log 2>&1
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/r2_1/bench_c5.log 2>&1
timeout 600 python bench.py --steps 20 --warmup 5 --config c3 --no-cpu-baseline > gpurun_out/r2_1/bench_c3.log 2>&1
timeout 300 python bench.py --steps 20 --warmup 5 --config c2 --no-cpu-baseline > gpurun_out/r2_1/bench_c2.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -rf -x > gpurun_out/r2_1/pytest_gpu.log 2>&1
echo done
