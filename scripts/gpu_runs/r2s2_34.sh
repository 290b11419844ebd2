# round 2 (re-entry): ncu of C2's free-warp kernel and C3's largest bundle kernel on the final tree,
# with their launch lists
set -x
mkdir -p gpurun_out/r2s2_34
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2s2_34/build.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2s2_34/launches_c2.csv python bench.py --steps 2 --warmup 3 --config c2 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cecjit -s 2 -c 1 -o gpurun_out/r2s2_34/prof_c2 python bench.py --steps 1 --warmup 3 --config c2 --no-cpu-baseline --e2e-steps 1 > gpurun_out/r2s2_34/ncu_c2.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2s2_34/launches_c3.csv python bench.py --steps 2 --warmup 3 --config c3 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:cecjit --launch-skip 60 -c 1 -o gpurun_out/r2s2_34/prof_c3 python bench.py --steps 1 --warmup 3 --config c3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/r2s2_34/ncu_c3.log 2>&1
echo done
