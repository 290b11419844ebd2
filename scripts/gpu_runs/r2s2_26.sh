# round 2 (re-entry): driver keeps its device contexts between check_miter calls; C4 flow x2; driver tests
set -x
mkdir -p gpurun_out/r2s2_26
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2s2_26/build.log 2>&1
for r in 1 2; do timeout 600 python scripts/c4_flow.py > gpurun_out/r2s2_26/c4_$r.jsonl 2>&1; done
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_local_pass.py -q -rf -k "driver or local" > gpurun_out/r2s2_26/pytest.log 2>&1
echo done
