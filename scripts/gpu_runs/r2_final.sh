# round 2, final verification on a fresh box: build + smoke, default bench (driver's command), reference arm,
# C1/C2/C2-bug/C3 benches, full GPU suite
set -x
mkdir -p gpurun_out/r2_final
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r2_final/smoke.log 2>&1
timeout 900 python3 bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/r2_final/bench_c5.log 2>&1
timeout 900 python3 bench.py --impl reference --gpus 1 --steps 20 --warmup 5 > gpurun_out/r2_final/bench_ref.log 2>&1
for c in c3 c2 c2bug c1; do timeout 600 python bench.py --steps 20 --warmup 5 --config $c --no-cpu-baseline > gpurun_out/r2_final/bench_$c.log 2>&1; done
timeout 2400 python -m pytest tests -m gpu -q -rf > gpurun_out/r2_final/pytest_gpu.log 2>&1
echo done
