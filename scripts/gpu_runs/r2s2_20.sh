# round 2 (re-entry): roofline over the window kernels' own event time, measured in a second pass of K steps with opt-in sweep events
set -x
mkdir -p gpurun_out/r2s2_20
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r2s2_20/smoke.log 2>&1
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/r2s2_20/bench_c5.log 2>&1
for c in c3 c2 c2bug c1; do timeout 600 python bench.py --steps 20 --warmup 5 --config $c --no-cpu-baseline > gpurun_out/r2s2_20/bench_$c.log 2>&1; done
timeout 900 python -m pytest tests/test_gpu_parity.py -q -rf -k "reload or plan_rerun or split or sweep_timing" > gpurun_out/r2s2_20/pytest.log 2>&1
echo done
