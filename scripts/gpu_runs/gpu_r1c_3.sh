# round 1c: peer-memory a10 (NEXT-4) tests on B200 + regression of parity + bench
mkdir -p gpurun_out/c3
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c3/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_peer.py -q -rf -x > gpurun_out/c3/peer.log 2>&1
timeout 1200 python -m pytest tests -q -m gpu -rf -x --deselect tests/test_gpu_peer.py > gpurun_out/c3/pytest.log 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/c3/bench.log 2>&1
echo done
