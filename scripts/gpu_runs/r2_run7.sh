# round 2, run 7: per-group timing of C3 and C2 plans; launch list of C3; ncu of C2 kernel (dual-pipe)
set -x
mkdir -p gpurun_out/r2_7
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2_7/build.log 2>&1
timeout 600 python scripts/profile_groups.py c3 > gpurun_out/r2_7/groups_c3.log 2>&1
timeout 600 python scripts/profile_groups.py c2 > gpurun_out/r2_7/groups_c2.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2_7/launches_c3.csv python bench.py --config c3 --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cecjit -s 3 -c 1 -o gpurun_out/r2_7/prof_c2 python bench.py --config c2 --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/r2_7/ncu_c2.log 2>&1
echo done
