# round 1c: C2/C5 block-sync vs warp-independent JIT, 256-thread blocks
mkdir -p gpurun_out/c15
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c15/build.log 2>&1
timeout 300 python bench.py --no-cpu-baseline --config c2 --e2e-steps 1 > gpurun_out/c15/c2_base.log 2>&1
CEC_JIT_SYNC=0 CEC_JIT_SPLICE=0 timeout 300 python bench.py --no-cpu-baseline --config c2 --e2e-steps 1 > gpurun_out/c15/c2_sync0.log 2>&1
CEC_JIT_THREADS=256 CEC_JIT_MINB=2 timeout 300 python bench.py --no-cpu-baseline --config c2 --e2e-steps 1 > gpurun_out/c15/c2_t256.log 2>&1
CEC_JIT_THREADS=128 CEC_JIT_MINB=4 timeout 300 python bench.py --no-cpu-baseline --config c2 --e2e-steps 1 > gpurun_out/c15/c2_t128.log 2>&1
CEC_JIT_THREADS=256 CEC_JIT_MINB=2 timeout 300 python bench.py --no-cpu-baseline --config c3 --e2e-steps 1 > gpurun_out/c15/c3_t256.log 2>&1
CEC_JIT_THREADS=256 CEC_JIT_MINB=2 timeout 300 python bench.py --no-cpu-baseline --config c5 --e2e-steps 1 > gpurun_out/c15/c5_t256.log 2>&1
echo done
