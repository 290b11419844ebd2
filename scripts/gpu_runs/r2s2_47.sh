# round 2 (re-entry): flat hash maps in the routing of pairs to windows: parity + C3/C5 call timing
set -x
mkdir -p gpurun_out/r2s2_47
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2s2_47/build.log 2>&1
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edge.py -q -rf -k "c3 or c5_full or cone or split or fuzz_tiny or invariance or pipelined or reload" > gpurun_out/r2s2_47/pytest.log 2>&1
timeout 300 python scripts/time_plan.py c3 5 > gpurun_out/r2s2_47/c3.log 2>&1
timeout 300 python scripts/time_plan.py c5 4 > gpurun_out/r2s2_47/c5.log 2>&1
echo done
