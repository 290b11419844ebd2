mkdir -p gpurun_out/t4
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/t4/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_reduce.py tests/test_gpu_classes.py tests/test_driver_host.py -q -m gpu -rf > gpurun_out/t4/pytest_new.log 2>&1
timeout 1200 python scripts/bench_flow.py --configs c2,c3,c5 > gpurun_out/t4/flow.jsonl 2> gpurun_out/t4/flow.err
timeout 600 python scripts/c4_flow.py > gpurun_out/t4/c4_flow.jsonl 2>&1
echo done
