# round 2, run 28: default bench with the all-core cpu baseline, reference arm, new local-check JIT test
set -x
mkdir -p gpurun_out/r2_28
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r2_28/smoke.log 2>&1
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/r2_28/bench_c5.log 2>&1
timeout 600 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/r2_28/bench_ref.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -rf -k "local_checks" > gpurun_out/r2_28/pytest_local.log 2>&1
echo done
