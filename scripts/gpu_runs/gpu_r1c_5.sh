# round 1c: peer-memory a10 tests (child processes with 32 connections)
mkdir -p gpurun_out/c5
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c5/build.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_peer.py -q -rf > gpurun_out/c5/peer.log 2>&1
echo done
