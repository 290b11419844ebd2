# round 1 (re-entry): rebuild, smoke, full GPU test suite, default bench + reference arm, launch list, ncu full of the JIT kernel
set -x
mkdir -p gpurun_out
nvidia-smi > gpurun_out/smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/bench_c5.log 2>&1
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu -rf > gpurun_out/pytest_gpu.log 2>&1
timeout 600 python bench.py --config c3 --no-cpu-baseline > gpurun_out/bench_c3.log 2>&1
timeout 300 python bench.py --config c2 --no-cpu-baseline > gpurun_out/bench_c2.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/b_ncu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cecjit -s 1 -c 1 -o gpurun_out/prof_jit_c5 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/ncu_full_c5.log 2>&1
echo done
