# round 1d (re-entry): verify the restored tree on a fresh B200: build, smoke, GPU tests, default bench, reference arm
mkdir -p gpurun_out/d1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/d1/build.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/d1/smoke.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu -rf > gpurun_out/d1/pytest.log 2>&1
timeout 900 python bench.py > gpurun_out/d1/bench_default.log 2>&1
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/d1/bench_ref.log 2>&1
for c in c3 c2; do timeout 600 python bench.py --no-cpu-baseline --config $c > gpurun_out/d1/bench_$c.log 2>&1; done
echo done
