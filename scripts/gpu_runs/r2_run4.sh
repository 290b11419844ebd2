# round 2, run 4: ncu full of C5's largest random-type kernel (third cecjit launch) under mapping mode 2,
# mode 3 with input masks only, and mode 3 with word-uniform node masks (default)
set -x
mkdir -p gpurun_out/r2_4
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2_4/build.log 2>&1
N="ncu --set full --clock-control none --import-source on -k regex:cecjit -s 2 -c 1"
B="python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1"
CEC_JIT_FUSE=2 timeout 900 $N -o gpurun_out/r2_4/prof_m2 $B > gpurun_out/r2_4/ncu_m2.log 2>&1
CEC_MAP_WU_NODES=0 timeout 900 $N -o gpurun_out/r2_4/prof_m3in $B > gpurun_out/r2_4/ncu_m3in.log 2>&1
timeout 900 $N -o gpurun_out/r2_4/prof_m3wu $B > gpurun_out/r2_4/ncu_m3wu.log 2>&1
CEC_TIMING=1 timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 3 > gpurun_out/r2_4/timing_c5.log 2>&1
echo done
