# round 2 (re-entry): worker-pool spin A/B (CEC_POOL_SPIN = 0 / 1024 / 4096 pause iterations)
set -x
mkdir -p gpurun_out/r2s2_12
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2s2_12/build.log 2>&1
for sp in 0 1024 4096; do
  CEC_POOL_SPIN=$sp timeout 300 python scripts/time_plan.py c3 5 > gpurun_out/r2s2_12/c3_$sp.log 2>&1
  CEC_POOL_SPIN=$sp timeout 300 python scripts/time_plan.py c5 3 > gpurun_out/r2s2_12/c5_$sp.log 2>&1
  CEC_POOL_SPIN=$sp timeout 600 python scripts/c4_flow.py > gpurun_out/r2s2_12/c4_$sp.log 2>&1
done
echo done
