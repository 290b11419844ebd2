# round 1c: C2 launch list + ncu full of its JIT kernel (256x2 block shape)
mkdir -p gpurun_out/c20
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c20/build.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/c20/launches_c2.csv python bench.py --config c2 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/c20/b_ncu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cecjit -s 3 -c 1 -o gpurun_out/c20/prof_c2 python bench.py --config c2 --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/c20/ncu_c2.log 2>&1
echo done
