# round 2 (re-entry): shard+split test; C4 flow local-pass timing with the mask cut path
set -x
mkdir -p gpurun_out/r2s2_25
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2s2_25/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -rf -k "shard_emulation" > gpurun_out/r2s2_25/pytest.log 2>&1
CEC_TIMING_LOCAL=1 timeout 600 python scripts/c4_flow.py > gpurun_out/r2s2_25/c4.jsonl 2> gpurun_out/r2s2_25/c4.err
CEC_CUTS_LISTS=1 CEC_TIMING_LOCAL=1 timeout 600 python scripts/c4_flow.py > gpurun_out/r2s2_25/c4_lists.jsonl 2> gpurun_out/r2s2_25/c4_lists.err
echo done
