# round 1c: final-state evidence: full GPU suite, smoke, default bench, reference arm, flow rows (c3, c5, c4), C3/C2 benches
mkdir -p gpurun_out/c25
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c25/build.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/c25/smoke.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu -rf > gpurun_out/c25/pytest.log 2>&1
timeout 600 python bench.py > gpurun_out/c25/bench.log 2>&1
timeout 600 python bench.py --impl reference > gpurun_out/c25/bench_ref.log 2>&1
timeout 600 python bench.py --no-cpu-baseline --config c3 > gpurun_out/c25/bench_c3.log 2>&1
timeout 600 python bench.py --no-cpu-baseline --config c2 > gpurun_out/c25/bench_c2.log 2>&1
timeout 900 python scripts/bench_flow.py --configs c3,c5,c4 > gpurun_out/c25/bench_flow.log 2>&1
echo done
