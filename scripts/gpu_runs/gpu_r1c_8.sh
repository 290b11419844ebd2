# round 1c: bench.py under torchrun with 2/4 ranks emulated on the one GPU (peer reduction, gloo PG)
mkdir -p gpurun_out/c8
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c8/build.log 2>&1
BENCH_SAME_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --steps 3 --warmup 3 --config c2bug > gpurun_out/c8/tr2_c2bug.log 2>&1
BENCH_SAME_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 4 --master-addr 127.0.0.1 --master-port 29512 bench.py --gpus 4 --steps 3 --warmup 3 > gpurun_out/c8/tr4_c5.log 2>&1
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29513 bench.py --gpus 1 --steps 3 --warmup 3 --config c2 > gpurun_out/c8/tr1_c2.log 2>&1
echo done
