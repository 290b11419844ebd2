# round 2 (re-entry): torchrun emulation of the multi-rank bench on ONE B200 (host barriers, gloo):
# the N > 1 path of bench.py with the kernel-time pass and the SURVEY record; reference arm at N = 2
set -x
mkdir -p gpurun_out/r2s2_48
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2s2_48/build.log 2>&1
BENCH_SAME_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29561 bench.py --gpus 2 --steps 3 --warmup 3 --config c2bug > gpurun_out/r2s2_48/tr2_c2bug.log 2>&1
BENCH_SAME_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 4 --master-addr 127.0.0.1 --master-port 29562 bench.py --gpus 4 --steps 3 --warmup 3 > gpurun_out/r2s2_48/tr4_c5.log 2>&1
BENCH_SAME_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29563 bench.py --impl reference --gpus 2 --steps 2 --warmup 3 > gpurun_out/r2s2_48/tr2_ref.log 2>&1
echo done
