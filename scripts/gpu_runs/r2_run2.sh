# round 2, run 2: dual-pipe cells (mapping mode 3: LOP3 + IMAD) vs mode 2 on C5/C3/C2; GPU tests
set -x
mkdir -p gpurun_out/r2_2
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r2_2/smoke.log 2>&1
B="python bench.py --steps 20 --warmup 5 --no-cpu-baseline"
timeout 900 $B > gpurun_out/r2_2/bench_c5_m3.log 2>&1
CEC_JIT_FUSE=2 timeout 900 $B > gpurun_out/r2_2/bench_c5_m2.log 2>&1
timeout 600 $B --config c3 > gpurun_out/r2_2/bench_c3_m3.log 2>&1
timeout 300 $B --config c2 > gpurun_out/r2_2/bench_c2_m3.log 2>&1
CEC_JIT_FUSE=2 timeout 300 $B --config c2 > gpurun_out/r2_2/bench_c2_m2.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q -rf -x > gpurun_out/r2_2/pytest_gpu.log 2>&1
echo done
