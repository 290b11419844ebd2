# tuning: exact-area mapping on C5/C2; small-window JIT config on C2; C3 per-group times and JIT threshold
mkdir -p gpurun_out/t2
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/t2/build.log 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/t2/c5.log 2>&1
for v in "" "CEC_JIT_SYNC=0" "CEC_JIT_THREADS=256" "CEC_JIT_THREADS=256 CEC_JIT_SYNC=0" "CEC_JIT_THREADS=384 CEC_JIT_SYNC=0" "CEC_JIT_THREADS=1024" "CEC_JIT_THREADS=128 CEC_JIT_SYNC=0 CEC_JIT_MINB=2"; do
  echo "== $v" >> gpurun_out/t2/c2.log
  env $v timeout 300 python bench.py --config c2 --no-cpu-baseline --e2e-steps 3 2>&1 | tail -1 >> gpurun_out/t2/c2.log
done
timeout 600 python scripts/profile_groups.py c3 > gpurun_out/t2/c3_groups.log 2>&1
for t in 2097152 4194304; do
  echo "== $t" >> gpurun_out/t2/c3.log
  CEC_JIT_MIN_NODE_WORDS=$t timeout 600 python bench.py --config c3 --no-cpu-baseline --e2e-steps 3 2>&1 | tail -1 >> gpurun_out/t2/c3.log
done
echo done
