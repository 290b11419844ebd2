# round 1c: cooperative single-launch partial simulation (NEXT-2): tests + flow rows
mkdir -p gpurun_out/c23
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c23/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_classes.py tests/test_gpu_reduce.py tests/test_gpu_parity.py -q -m gpu -rf -k "classes or random or patterns or reduce or driver" > gpurun_out/c23/pytest.log 2>&1
timeout 900 python scripts/bench_flow.py > gpurun_out/c23/bench_flow.log 2>&1
CEC_RS_LEVEL_LAUNCHES=1 timeout 900 python scripts/bench_flow.py > gpurun_out/c23/bench_flow_levels.log 2>&1
echo done
