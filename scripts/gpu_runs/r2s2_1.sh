# round 2 (re-entry session): sanity on a fresh box after the container was re-created:
# build + smoke, default C5 bench, C3/C2 benches, host phase timing of C3
set -x
mkdir -p gpurun_out/r2s2_1
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r2s2_1/smoke.log 2>&1
timeout 900 python3 bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/r2s2_1/bench_c5.log 2>&1
for c in c3 c2; do timeout 600 python bench.py --steps 20 --warmup 5 --config $c --no-cpu-baseline > gpurun_out/r2s2_1/bench_$c.log 2>&1; done
timeout 600 python scripts/time_plan.py c3 4 > gpurun_out/r2s2_1/time_plan_c3.log 2>&1
echo done
