# round 2 (re-entry): GC paused during the flow: C4 flow x2 processes, C3/C5 calls
set -x
mkdir -p gpurun_out/r2s2_14
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2s2_14/build.log 2>&1
for r in 1 2; do timeout 600 python scripts/c4_flow.py > gpurun_out/r2s2_14/c4_$r.log 2>&1; done
timeout 300 python scripts/time_plan.py c3 5 > gpurun_out/r2s2_14/c3.log 2>&1
timeout 300 python scripts/time_plan.py c5 3 > gpurun_out/r2s2_14/c5.log 2>&1
timeout 900 python -m pytest tests/test_gpu_local_pass.py tests/test_gpu_parity.py -q -rf -k "local or cut or c4 or driver" > gpurun_out/r2s2_14/pytest.log 2>&1
echo done
