# work-based bundling + hoisted input words: parity suite, C5/C2/C3 bench, C3 JIT threshold sweep
mkdir -p gpurun_out/t7
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/t7/smoke.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -m gpu -rf -x > gpurun_out/t7/pytest_gpu.log 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/t7/c5.log 2>&1
timeout 300 python bench.py --config c2 --no-cpu-baseline > gpurun_out/t7/c2.log 2>&1
for t in 8388608 2097152 1048576; do
  echo "== $t" >> gpurun_out/t7/c3.log
  CEC_JIT_MIN_NODE_WORDS=$t timeout 900 python bench.py --config c3 --no-cpu-baseline 2>&1 | tail -1 >> gpurun_out/t7/c3.log
done
echo done
