# round 2 (re-entry): peer tests with host barriers (no kernels waiting on one another on one GPU),
# the device barrier's timeout path alone, split-pipelining parity, torchrun emulation of the bench
set -x
mkdir -p gpurun_out/r2s2_5
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2s2_5/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_peer.py -q -rf > gpurun_out/r2s2_5/pytest_peer.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -rf -k "split or c3_full or pipelined" > gpurun_out/r2s2_5/pytest_split.log 2>&1
BENCH_SAME_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29551 bench.py --gpus 2 --steps 3 --warmup 3 --config c2bug > gpurun_out/r2s2_5/tr2_c2bug.log 2>&1
echo done
