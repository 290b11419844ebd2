mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for T in 8388608 2097152 1048576; do for S in 4 8 16 32; do
 echo "T=$T S=$S" >> gpurun_out/sweep_c3.log
 CEC_JIT_MIN_NODE_WORDS=$T CEC_SIDE_STREAMS=$S timeout 600 python bench.py --config c3 --no-cpu-baseline --e2e-steps 1 2>&1 | tail -1 >> gpurun_out/sweep_c3.log
done; done
echo done
