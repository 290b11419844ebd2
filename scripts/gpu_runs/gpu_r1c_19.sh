# round 1c: parallel interpreter-program copy, smoke with a JIT case: full suite + smoke + benches
mkdir -p gpurun_out/c19
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c19/build.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/c19/smoke.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu -rf > gpurun_out/c19/pytest.log 2>&1
timeout 600 python bench.py > gpurun_out/c19/bench.log 2>&1
timeout 600 python bench.py --no-cpu-baseline --config c3 > gpurun_out/c19/bench_c3.log 2>&1
echo done
