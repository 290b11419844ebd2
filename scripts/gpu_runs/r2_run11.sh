# round 2, run 11: C3 bundling sweep (standalone threshold, bundle size) under the dual-pipe mapping
set -x
mkdir -p gpurun_out/r2_11
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2_11/build.log 2>&1
B="python bench.py --config c3 --steps 10 --warmup 4 --no-cpu-baseline --e2e-steps 1"
timeout 600 $B > gpurun_out/r2_11/base.log 2>&1
CEC_BUNDLE_BELOW=4294967296 timeout 600 $B > gpurun_out/r2_11/below32.log 2>&1
CEC_BUNDLE_BELOW=8589934592 timeout 600 $B > gpurun_out/r2_11/below33.log 2>&1
CEC_BUNDLE_BELOW=34359738368 timeout 600 $B > gpurun_out/r2_11/below35.log 2>&1
CEC_BUNDLE_MAX=8 timeout 600 $B > gpurun_out/r2_11/max8.log 2>&1
CEC_BUNDLE_MAX=12 timeout 600 $B > gpurun_out/r2_11/max12.log 2>&1
CEC_BUNDLE_MAX=48 timeout 600 $B > gpurun_out/r2_11/max48.log 2>&1
echo done
