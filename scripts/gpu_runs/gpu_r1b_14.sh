mkdir -p gpurun_out/t14
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/t14/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_edge.py -q -m gpu -rf > gpurun_out/t14/pytest_edge.log 2>&1
echo done
