# round 2, run 5: ALU/FMA pipe co-issue microbenchmark; IMAD cell price sweep on C5; mapping-mode parity test
set -x
mkdir -p gpurun_out/r2_5
nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/pipes scripts/pipes.cu && timeout 120 /tmp/pipes > gpurun_out/r2_5/pipes.json 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2_5/build.log 2>&1
B="python bench.py --steps 10 --warmup 4 --no-cpu-baseline --e2e-steps 1"
for b in 0.25 0.5 0.75; do CEC_MAP_IMAD=$b timeout 600 $B > gpurun_out/r2_5/bench_c5_b$b.log 2>&1; done
timeout 900 python -m pytest tests/test_gpu_parity.py -q -rf -x -k "cell_mappings" > gpurun_out/r2_5/pytest_modes.log 2>&1
echo done
