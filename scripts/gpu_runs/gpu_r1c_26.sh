# round 1c: programmatic dependent launch of the first JIT kernel after the reset kernel: tests + A/B
mkdir -p gpurun_out/c26
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c26/build.log 2>&1
for c in c2 c2bug c5 c3 c1; do
  timeout 600 python bench.py --no-cpu-baseline --config $c --e2e-steps 1 > gpurun_out/c26/bench_$c.log 2>&1
  CEC_NO_PDL=1 timeout 600 python bench.py --no-cpu-baseline --config $c --e2e-steps 1 > gpurun_out/c26/bench_${c}_nopdl.log 2>&1
done
timeout 1500 python -m pytest tests -q -m gpu -rf > gpurun_out/c26/pytest.log 2>&1
echo done
