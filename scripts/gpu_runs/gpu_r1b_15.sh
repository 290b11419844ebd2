mkdir -p gpurun_out/t15
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/t15/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -rf -k "shard or nccl or pipelined or invariance" > gpurun_out/t15/pytest.log 2>&1
echo done
