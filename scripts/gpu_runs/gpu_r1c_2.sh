# round 1c: strong-scaling emulation of C5 (each rank's shard alone) + e2e phase timing
mkdir -p gpurun_out/c2
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c2/build.log 2>&1
timeout 900 python scripts/scale_emulate.py > gpurun_out/c2/scale.jsonl 2> gpurun_out/c2/scale.err
CEC_TIMING=1 timeout 600 python bench.py --no-cpu-baseline --steps 3 --e2e-steps 5 > gpurun_out/c2/c5_timing.log 2>&1
echo done
