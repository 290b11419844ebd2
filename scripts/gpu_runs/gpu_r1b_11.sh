mkdir -p gpurun_out/t11
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/t11/build.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cecjit -s 3 -c 1 -o gpurun_out/t11/prof_c2 python bench.py --config c2 --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/t11/ncu_c2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cecjit -s 40 -c 1 -o gpurun_out/t11/prof_c3 python bench.py --config c3 --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/t11/ncu_c3.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/t11/c2_launches.csv python bench.py --config c2 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1
echo done
