# round 2, run 21: checkpoint after the barrier-cadence change: default benches, GPU suite, launch list + ncu of the big C5 kernel
set -x
mkdir -p gpurun_out/r2_21
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r2_21/smoke.log 2>&1
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/r2_21/bench_c5.log 2>&1
timeout 600 python bench.py --steps 20 --warmup 5 --config c3 --no-cpu-baseline > gpurun_out/r2_21/bench_c3.log 2>&1
timeout 300 python bench.py --steps 20 --warmup 5 --config c2 --no-cpu-baseline > gpurun_out/r2_21/bench_c2.log 2>&1
timeout 300 python bench.py --steps 20 --warmup 5 --config c2bug --no-cpu-baseline > gpurun_out/r2_21/bench_c2bug.log 2>&1
timeout 300 python bench.py --steps 20 --warmup 5 --config c1 --no-cpu-baseline > gpurun_out/r2_21/bench_c1.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2_21/launches_c5.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cecjit -s 2 -c 1 -o gpurun_out/r2_21/prof_c5 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/r2_21/ncu_c5.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -rf > gpurun_out/r2_21/pytest_gpu.log 2>&1
echo done
