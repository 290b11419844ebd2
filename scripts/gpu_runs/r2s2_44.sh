# round 2 (re-entry): small interpreter windows scheduled directly (no separate liveness count) -- measured slower (C3 call 14.0 vs 12.8-13.3 ms), reverted
set -x
mkdir -p gpurun_out/r2s2_44
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2s2_44/build.log 2>&1
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edge.py -q -rf -k "c3 or split or bundles or fuzz_tiny or c1 or local or small_multipliers or cone" > gpurun_out/r2s2_44/pytest.log 2>&1
timeout 900 python scripts/fuzz_jit.py --engine auto --seeds 300 --start 2000 > gpurun_out/r2s2_44/fuzz_auto.jsonl 2>&1
timeout 900 python scripts/fuzz_jit.py --engine interp --seeds 300 --start 3000 > gpurun_out/r2s2_44/fuzz_interp.jsonl 2>&1
timeout 300 python scripts/time_plan.py c3 5 > gpurun_out/r2s2_44/c3.log 2>&1
timeout 600 python bench.py --steps 20 --warmup 5 --config c3 --no-cpu-baseline > gpurun_out/r2s2_44/bench_c3.log 2>&1
echo done
