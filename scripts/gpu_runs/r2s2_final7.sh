# round 2 (re-entry session) final verification #7 (final tree): build + smoke, driver bench commands, C3/C2/C2-bug/C1, C4 flow, launch list + ncu of the largest C5 kernel, full GPU suite
# commands (ours, reference arm), C3/C2/C2-bug/C1 benches, C4 flow, launch list + ncu --set full of
# the largest C5 kernel, full GPU suite
set -x
mkdir -p gpurun_out/r2s2_final7
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r2s2_final7/smoke.log 2>&1
timeout 900 python3 bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/r2s2_final7/bench_c5.log 2>&1
timeout 900 python3 bench.py --impl reference --gpus 1 --steps 20 --warmup 5 > gpurun_out/r2s2_final7/bench_ref.log 2>&1
for c in c3 c2 c2bug c1; do timeout 600 python bench.py --steps 20 --warmup 5 --config $c --no-cpu-baseline > gpurun_out/r2s2_final7/bench_$c.log 2>&1; done
timeout 600 python scripts/c4_flow.py > gpurun_out/r2s2_final7/c4_flow.jsonl 2> gpurun_out/r2s2_final7/c4_flow.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2s2_final7/launches_c5.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cecjit -s 2 -c 1 -o gpurun_out/r2s2_final7/prof_c5 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/r2s2_final7/ncu_c5.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -rf > gpurun_out/r2s2_final7/pytest_gpu.log 2>&1
echo done
