set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
B="python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1"
timeout 600 $B > gpurun_out/f_c5.log 2>&1
CEC_JIT_FUSE=0 timeout 600 $B > gpurun_out/f_c5_nofuse.log 2>&1
timeout 600 $B --config c2 > gpurun_out/f_c2.log 2>&1
timeout 900 $B --config c3 > gpurun_out/f_c3.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -rf > gpurun_out/pytest_gpu.log 2>&1
timeout 900 python scripts/c4_flow.py > gpurun_out/c4_flow.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/b_ncu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cecjit -s 1 -c 1 -o gpurun_out/prof_jit_c5_fused python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/ncu_full_c5.log 2>&1
echo done
