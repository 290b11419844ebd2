# round 2, run 29: torchrun emulation of the multi-rank bench path on ONE B200 (ranks time-slice the GPU;
# checks peer setup, sharded free-warp/dual-pipe plans, fused min, parity), and the peer tests
set -x
mkdir -p gpurun_out/r2_29
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2_29/build.log 2>&1
BENCH_SAME_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29541 bench.py --gpus 2 --steps 3 --warmup 3 --config c2bug > gpurun_out/r2_29/tr2_c2bug.log 2>&1
BENCH_SAME_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 3 --master-addr 127.0.0.1 --master-port 29542 bench.py --gpus 3 --steps 3 --warmup 3 --config c2 > gpurun_out/r2_29/tr3_c2.log 2>&1
BENCH_SAME_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 4 --master-addr 127.0.0.1 --master-port 29543 bench.py --gpus 4 --steps 3 --warmup 3 > gpurun_out/r2_29/tr4_c5.log 2>&1
BENCH_SAME_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29544 bench.py --impl reference --gpus 2 --steps 2 --warmup 3 > gpurun_out/r2_29/tr2_ref.log 2>&1
timeout 900 python -m pytest tests/test_gpu_peer.py -q -rf > gpurun_out/r2_29/pytest_peer.log 2>&1
echo done
