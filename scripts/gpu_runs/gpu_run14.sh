set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/smoke.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2.csv python bench.py --config c2 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/b_ncu_c2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cecjit -s 3 -c 1 -o gpurun_out/prof_c2_area python bench.py --config c2 --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/ncu_c2.log 2>&1
echo done
