set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
B="python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1"
timeout 300 $B --engine 1 --config c2 > gpurun_out/i_c2.log 2>&1
timeout 600 $B --engine 1 > gpurun_out/i_c5.log 2>&1
timeout 900 $B --config c3 > gpurun_out/c3.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -rf > gpurun_out/pytest_gpu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:interp -s 3 -c 1 -o gpurun_out/prof_interp_c2 python bench.py --config c2 --engine 1 --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/ncu_full_c2i.log 2>&1
echo done
