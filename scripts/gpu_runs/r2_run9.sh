# round 2, run 9: checkpoint — full GPU suite, default benches C5/C3/C2 with the reference arm, scaling emulation
set -x
mkdir -p gpurun_out/r2_9
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r2_9/smoke.log 2>&1
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/r2_9/bench_c5.log 2>&1
timeout 600 python bench.py --steps 20 --warmup 5 --config c3 --no-cpu-baseline > gpurun_out/r2_9/bench_c3.log 2>&1
timeout 300 python bench.py --steps 20 --warmup 5 --config c2 --no-cpu-baseline > gpurun_out/r2_9/bench_c2.log 2>&1
timeout 600 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/r2_9/bench_ref.log 2>&1
timeout 900 python scripts/scale_emulate.py > gpurun_out/r2_9/scale_emulated.jsonl 2>gpurun_out/r2_9/scale.err
timeout 2400 python -m pytest tests -m gpu -q -rf > gpurun_out/r2_9/pytest_gpu.log 2>&1
echo done
