# NEXT-2/NEXT-3 GPU parity (classes, reduction), driver tests, C4 flow, C5 bench with host phase timing
mkdir -p gpurun_out/t3
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/t3/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_reduce.py tests/test_gpu_classes.py tests/test_driver_host.py -q -m gpu -rf -x > gpurun_out/t3/pytest_new.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -rf -k "driver" > gpurun_out/t3/pytest_driver.log 2>&1
timeout 600 python scripts/c4_flow.py > gpurun_out/t3/c4_flow.jsonl 2>&1
CEC_TIMING=1 timeout 600 python bench.py --no-cpu-baseline --steps 3 --e2e-steps 3 > gpurun_out/t3/c5_timing.log 2>&1
nproc > gpurun_out/t3/nproc.txt
echo done
