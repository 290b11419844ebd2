# round 2 (re-entry): device AIG buffers kept across cec_reload_aig; C4 flow x3 processes; flow tests
set -x
mkdir -p gpurun_out/r2s2_23
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2s2_23/build.log 2>&1
for r in 1 2 3; do timeout 600 python scripts/c4_flow.py > gpurun_out/r2s2_23/c4_$r.jsonl 2>&1; done
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_classes.py tests/test_gpu_reduce.py tests/test_gpu_local_pass.py -q -rf -k "reload or driver or classes or reduce or local" > gpurun_out/r2s2_23/pytest.log 2>&1
echo done
