# round 2, run 6: block shape / barrier cadence sweep of the C5 kernels under the dual-pipe mapping
set -x
mkdir -p gpurun_out/r2_6
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2_6/build.log 2>&1
B="python bench.py --steps 10 --warmup 4 --no-cpu-baseline --e2e-steps 1"
timeout 600 $B > gpurun_out/r2_6/base.log 2>&1
CEC_JIT_THREADS=384 CEC_JIT_MINB=1 timeout 600 $B > gpurun_out/r2_6/t384.log 2>&1
CEC_JIT_THREADS=256 CEC_JIT_MINB=1 timeout 600 $B > gpurun_out/r2_6/t256x1.log 2>&1
CEC_JIT_THREADS=640 CEC_JIT_MINB=1 timeout 600 $B > gpurun_out/r2_6/t640.log 2>&1
CEC_JIT_SYNC=256 timeout 600 $B > gpurun_out/r2_6/sync256.log 2>&1
CEC_JIT_SYNC=1024 timeout 600 $B > gpurun_out/r2_6/sync1024.log 2>&1
echo done
