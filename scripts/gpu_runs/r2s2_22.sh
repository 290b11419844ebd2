# round 2 (re-entry): CEX vectors from the compares' supports (no TFI walk in resolve_results)
set -x
mkdir -p gpurun_out/r2s2_22
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2s2_22/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edge.py -q -rf -k "fuzz or c2_full or pipelined or small_multipliers or cex or reload or c5_reduced or split" > gpurun_out/r2s2_22/pytest.log 2>&1
timeout 300 python scripts/time_plan.py c5 3 > gpurun_out/r2s2_22/c5.log 2>&1
echo done
