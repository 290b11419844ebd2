# round 1c: peer import checks P2P atomics by PCI bus id: peer tests + torchrun emulation
mkdir -p gpurun_out/c14
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c14/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_peer.py -q -rf > gpurun_out/c14/peer.log 2>&1
BENCH_SAME_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29521 bench.py --gpus 2 --steps 3 --warmup 3 --config c2bug > gpurun_out/c14/tr2_c2bug.log 2>&1
echo done
