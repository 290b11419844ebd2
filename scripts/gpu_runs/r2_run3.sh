# round 2, run 3: dual-pipe cells with word-uniform NODES as m (default) vs inputs only; ncu of C5
set -x
mkdir -p gpurun_out/r2_3
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r2_3/smoke.log 2>&1
B="python bench.py --steps 20 --warmup 5 --no-cpu-baseline"
timeout 900 $B > gpurun_out/r2_3/bench_c5_wu.log 2>&1
CEC_MAP_WU_NODES=0 timeout 900 $B > gpurun_out/r2_3/bench_c5_inputs.log 2>&1
timeout 600 $B --config c3 > gpurun_out/r2_3/bench_c3_wu.log 2>&1
timeout 300 $B --config c2 > gpurun_out/r2_3/bench_c2_wu.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2_3/launches_c5.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cecjit -s 1 -c 1 -o gpurun_out/r2_3/prof_c5 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/r2_3/ncu_c5.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q -rf -x -k "parity or edge or jit" > gpurun_out/r2_3/pytest_gpu.log 2>&1
echo done
