# round 1c: peer-memory a10 tests (multi-process IPC emulation) + C5 golden copies [160, 256) on the host cores
mkdir -p gpurun_out/c6
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c6/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_peer.py -q -rf > gpurun_out/c6/peer.log 2>&1
GOLDEN_PARTIAL=gpurun_out/c6/c5_partial_box.jsonl timeout 2400 python scripts/make_golden_c5.py 16 160 256 > gpurun_out/c6/golden.log 2>&1
echo done
