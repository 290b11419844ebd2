# round 1c: per-kernel block shape (256x2 for bodies <= 4096 ANDs): benches + full GPU suite
mkdir -p gpurun_out/c16
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c16/build.log 2>&1
for c in c5 c3 c2 c2bug c1; do
  timeout 600 python bench.py --no-cpu-baseline --config $c > gpurun_out/c16/bench_$c.log 2>&1
done
timeout 1500 python -m pytest tests -q -m gpu -rf > gpurun_out/c16/pytest.log 2>&1
echo done
