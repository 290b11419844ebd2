# round 1c: peer-memory a10 tests (warmed contexts)
mkdir -p gpurun_out/c4
nproc > gpurun_out/c4/nproc.txt; lscpu | head -20 >> gpurun_out/c4/nproc.txt
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c4/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_peer.py -q -rf > gpurun_out/c4/peer.log 2>&1
echo done
