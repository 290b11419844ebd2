mkdir -p gpurun_out/t12
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/t12/smoke.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_sanitizer.py -q -m gpu -rf -x > gpurun_out/t12/pytest.log 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/t12/c5.log 2>&1
timeout 900 python bench.py --config c3 --no-cpu-baseline > gpurun_out/t12/c3.log 2>&1
timeout 300 python bench.py --config c2 --no-cpu-baseline > gpurun_out/t12/c2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cecjit -s 3 -c 1 -o gpurun_out/t12/prof_c2 python bench.py --config c2 --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/t12/ncu_c2.log 2>&1
echo done
