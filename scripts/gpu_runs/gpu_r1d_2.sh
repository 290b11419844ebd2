# round 1d: per-phase host timings of the e2e call (C3, C5) to find the host-prep hot spots
mkdir -p gpurun_out/d2
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/d2/build.log 2>&1
for c in c3 c5; do CEC_TIMING=1 timeout 600 python bench.py --no-cpu-baseline --config $c --steps 3 --e2e-steps 3 > gpurun_out/d2/bench_$c.log 2>&1; done
nproc > gpurun_out/d2/nproc.txt
echo done
