# round 2 (re-entry): C4 flow with parallel small levels + parallel common cuts (CEC_CUT_PAR_MIN=8: old)
set -x
mkdir -p gpurun_out/r2s2_10
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2s2_10/build.log 2>&1
CEC_TIMING_LOCAL=1 timeout 600 python scripts/c4_flow.py > gpurun_out/r2s2_10/c4.log 2> gpurun_out/r2s2_10/c4.err
CEC_CUT_PAR_MIN=8 timeout 600 python scripts/c4_flow.py > gpurun_out/r2s2_10/c4_old.log 2> gpurun_out/r2s2_10/c4_old.err
timeout 1200 python -m pytest tests/test_gpu_local_pass.py tests/test_gpu_parity.py -q -rf -k "local or cut or c4 or driver" > gpurun_out/r2s2_10/pytest.log 2>&1
echo done
