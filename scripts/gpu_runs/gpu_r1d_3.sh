# round 1d: longest-first order of the parallel per-window planning (A/B vs FIFO via CEC_PLAN_FIFO=1) + GPU tests
mkdir -p gpurun_out/d3
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/d3/build.log 2>&1
for c in c3 c5; do
  for r in 1 2; do
    CEC_TIMING=1 timeout 600 python bench.py --no-cpu-baseline --config $c --steps 3 --e2e-steps 5 > gpurun_out/d3/bench_${c}_lpt_$r.log 2>&1
    CEC_PLAN_FIFO=1 CEC_TIMING=1 timeout 600 python bench.py --no-cpu-baseline --config $c --steps 3 --e2e-steps 5 > gpurun_out/d3/bench_${c}_fifo_$r.log 2>&1
  done
done
timeout 1500 python -m pytest tests -q -m gpu -rf > gpurun_out/d3/pytest.log 2>&1
echo done
