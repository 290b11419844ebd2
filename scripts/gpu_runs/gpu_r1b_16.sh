mkdir -p gpurun_out/t16
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/t16/build.log 2>&1
for K in 4 8 16; do
  echo "== $K" >> gpurun_out/t16/c5.log
  CEC_PIPELINE=$K timeout 600 python bench.py --no-cpu-baseline --steps 3 --e2e-steps 5 2>&1 | tail -1 >> gpurun_out/t16/c5.log
done
for K in 1 4; do
  echo "== $K" >> gpurun_out/t16/c3.log
  CEC_PIPELINE=$K timeout 600 python bench.py --config c3 --no-cpu-baseline --steps 3 --e2e-steps 5 2>&1 | tail -1 >> gpurun_out/t16/c3.log
done
echo done
