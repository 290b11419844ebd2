set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
B="python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1"
CEC_JIT_SYNC=1024 timeout 300 $B > gpurun_out/t_sync1024.log 2>&1
CEC_JIT_SYNC=2048 timeout 300 $B > gpurun_out/t_sync2048.log 2>&1
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/bench.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/b_ncu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cecjit -s 0 -c 1 -o gpurun_out/prof_jit_c5 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/ncu_full_c5.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -q -rf -k "driver" > gpurun_out/pytest_driver.log 2>&1
echo done
