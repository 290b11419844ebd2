# round 1c: regression (routing hash, C3 golden test), benches, reference arm, ncu launch list + full capture of the C5 kernel
mkdir -p gpurun_out/c10
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c10/build.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu -rf > gpurun_out/c10/pytest.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/c10/smoke.log 2>&1
timeout 600 python bench.py > gpurun_out/c10/bench.log 2>&1
timeout 600 python bench.py --no-cpu-baseline --config c3 > gpurun_out/c10/bench_c3.log 2>&1
timeout 600 python bench.py --no-cpu-baseline --config c2 > gpurun_out/c10/bench_c2.log 2>&1
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/c10/bench_ref.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/c10/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/c10/b_ncu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cecjit -s 1 -c 1 -o gpurun_out/c10/prof_jit_c5 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/c10/ncu_full_c5.log 2>&1
echo done
