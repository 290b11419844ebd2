# round 2 (re-entry): small configs: CUDA graph replay vs direct launches (CEC_NO_GRAPH=1)
set -x
mkdir -p gpurun_out/r2s2_17
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2s2_17/build.log 2>&1
for c in c2 c1 c2bug; do
  timeout 600 python bench.py --steps 50 --warmup 5 --config $c --no-cpu-baseline > gpurun_out/r2s2_17/bench_${c}_graph.log 2>&1
  CEC_NO_GRAPH=1 timeout 600 python bench.py --steps 50 --warmup 5 --config $c --no-cpu-baseline > gpurun_out/r2s2_17/bench_${c}_nograph.log 2>&1
done
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/r2s2_17/launches_c2.csv python bench.py --steps 3 --warmup 3 --config c2 --no-cpu-baseline > gpurun_out/r2s2_17/ncu_c2.log 2>&1
echo done
