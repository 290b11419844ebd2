set -x
mkdir -p gpurun_out
nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o gpurun_out/peaks scripts/peaks.cu && timeout 300 ./gpurun_out/peaks > gpurun_out/peaks.json 2> gpurun_out/peaks.err
( nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,power.draw --format=csv -lms 200 > gpurun_out/peaks_clk.csv & P=$!; sleep 0.1; timeout 300 ./gpurun_out/peaks > gpurun_out/peaks2.json; kill $P )
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -q -m gpu -x -k "rerun" > gpurun_out/test_rerun.log 2>&1
timeout 900 python bench.py --config c3 > gpurun_out/bench_c3.log 2>&1
CEC_NO_GRAPH=1 timeout 900 python bench.py --config c3 --no-cpu-baseline > gpurun_out/bench_c3_nograph.log 2>&1
timeout 900 python bench.py > gpurun_out/bench_c5.log 2>&1
timeout 900 python bench.py --config c2 --no-cpu-baseline > gpurun_out/bench_c2.log 2>&1
echo done
