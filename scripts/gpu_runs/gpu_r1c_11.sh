# round 1c: C3 per-group device times (serial launches), C4 flow, flow rows
mkdir -p gpurun_out/c11
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c11/build.log 2>&1
CEC_PROFILE_GROUPS=1 timeout 600 python bench.py --no-cpu-baseline --config c3 --steps 1 --e2e-steps 1 > gpurun_out/c11/c3_groups.log 2>&1
timeout 600 python scripts/c4_flow.py > gpurun_out/c11/c4_flow.log 2>&1
timeout 900 python scripts/bench_flow.py > gpurun_out/c11/bench_flow.log 2>&1
echo done
