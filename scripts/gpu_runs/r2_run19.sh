# round 2, run 19: in-body barrier cadence sweep for C5 (2 repetitions each)
set -x
mkdir -p gpurun_out/r2_19
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2_19/build.log 2>&1
B="python bench.py --steps 10 --warmup 4 --no-cpu-baseline --e2e-steps 1"
for r in 1 2; do for s in 512 1024 2048 4096; do CEC_JIT_SYNC=$s timeout 600 $B > gpurun_out/r2_19/sync${s}_$r.log 2>&1; done; done
echo done
