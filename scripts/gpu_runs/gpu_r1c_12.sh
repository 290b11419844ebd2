# round 1c: JIT fast body (accumulated compares, exact re-run on mismatch): tests + A/B benches
mkdir -p gpurun_out/c12
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c12/build.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu -rf -x > gpurun_out/c12/pytest.log 2>&1
for c in c5 c3 c2 c2bug; do
  timeout 600 python bench.py --no-cpu-baseline --config $c > gpurun_out/c12/bench_$c.log 2>&1
  CEC_JIT_ACC=0 timeout 600 python bench.py --no-cpu-baseline --config $c > gpurun_out/c12/bench_${c}_noacc.log 2>&1
done
echo done
