# round 1c: fast body v2 (rare path recomputes inputs): A/B benches + parity tests
mkdir -p gpurun_out/c13
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c13/build.log 2>&1
for c in c2 c5 c3 c2bug; do
  timeout 600 python bench.py --no-cpu-baseline --config $c --e2e-steps 1 > gpurun_out/c13/bench_$c.log 2>&1
done
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edge.py -q -m gpu -rf -x > gpurun_out/c13/pytest.log 2>&1
echo done
