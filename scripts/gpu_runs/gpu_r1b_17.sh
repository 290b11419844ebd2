mkdir -p gpurun_out/t17
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/t17/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu -rf -k "pipelined" > gpurun_out/t17/pytest.log 2>&1
CEC_TIMING=1 timeout 600 python bench.py --no-cpu-baseline --steps 3 --e2e-steps 5 > gpurun_out/t17/c5.log 2>&1
echo done
