# round 1c: peer timeout param + collective-safe bench setup: peer tests, torchrun emulation x2 (c2bug) and x4 (c5)
mkdir -p gpurun_out/c17
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c17/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_peer.py -q -rf > gpurun_out/c17/peer.log 2>&1
BENCH_SAME_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29531 bench.py --gpus 2 --steps 3 --warmup 3 --config c2bug > gpurun_out/c17/tr2_c2bug.log 2>&1
BENCH_SAME_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 4 --master-addr 127.0.0.1 --master-port 29532 bench.py --gpus 4 --steps 3 --warmup 3 > gpurun_out/c17/tr4_c5.log 2>&1
echo done
