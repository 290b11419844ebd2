# round 1d: new V4 closed-form own-index test (merged window + pext) on the GPU
mkdir -p gpurun_out/d4
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/d4/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_edge.py tests/test_gpu_parity.py -q -m gpu -rf > gpurun_out/d4/pytest.log 2>&1
echo done
