set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 1 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/torchrun1.log 2>&1
timeout 900 ncu --set full --clock-control none -k regex:simt_level -s 50 -c 1 -o gpurun_out/prof_simt_c5 python bench.py --engine 3 --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/ncu_simt.log 2>&1
timeout 900 python bench.py > gpurun_out/bench_final.log 2>&1
echo done
