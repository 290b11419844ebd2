# round 2 (re-entry): C3 split-pipelining threshold sweep (e2e through the public call)
set -x
mkdir -p gpurun_out/r2s2_4
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2s2_4/build.log 2>&1
for e in 0 24 26 28 30; do
  if [ $e = 0 ]; then v=0; else v=$(python -c "print(float(2**$e))"); fi
  CEC_PIPE_SPLIT=$v timeout 600 python scripts/time_plan.py c3 6 > gpurun_out/r2s2_4/time_plan_c3_$e.log 2>&1
done
echo done
