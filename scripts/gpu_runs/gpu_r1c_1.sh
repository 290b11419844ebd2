# round 1c: full verification of HEAD on B200 (gpu tests, smoke, default bench)
mkdir -p gpurun_out/c1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c1/build.log 2>&1
timeout 1200 python -m pytest tests -q -m gpu -rf -x > gpurun_out/c1/pytest.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/c1/smoke.log 2>&1
timeout 600 python bench.py > gpurun_out/c1/bench.log 2>&1
echo done
