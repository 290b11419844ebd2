# round 2, run 20: in-body barrier cadence 4096 / 8192 / none for C5; C3 and C2 at 4096
set -x
mkdir -p gpurun_out/r2_20
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2_20/build.log 2>&1
B="python bench.py --steps 10 --warmup 4 --no-cpu-baseline --e2e-steps 1"
for r in 1 2; do for s in 4096 8192 1000000; do CEC_JIT_SYNC=$s timeout 600 $B > gpurun_out/r2_20/sync${s}_$r.log 2>&1; done; done
CEC_JIT_SYNC=4096 timeout 600 $B --config c3 > gpurun_out/r2_20/c3_sync4096.log 2>&1
timeout 600 $B --config c3 > gpurun_out/r2_20/c3_sync512.log 2>&1
echo done
