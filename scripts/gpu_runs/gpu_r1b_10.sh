mkdir -p gpurun_out/t10
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/t10/smoke.log 2>&1
timeout 900 python -m pytest tests/test_gpu_local_pass.py tests/test_driver_host.py tests/test_gpu_reduce.py -q -m gpu -rf > gpurun_out/t10/pytest_new.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -rf -k "driver or local" > gpurun_out/t10/pytest_driver.log 2>&1
timeout 600 python scripts/c4_flow.py > gpurun_out/t10/c4_flow.jsonl 2>&1
echo done
