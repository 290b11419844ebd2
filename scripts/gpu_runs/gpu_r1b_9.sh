mkdir -p gpurun_out/t9
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/t9/smoke.log 2>&1
timeout 900 python bench.py --config c3 --no-cpu-baseline > gpurun_out/t9/c3.log 2>&1
timeout 600 python scripts/c4_flow.py > gpurun_out/t9/c4_flow.jsonl 2>&1
timeout 1200 python scripts/bench_flow.py --configs c4,c2,c3,c5 > gpurun_out/t9/flow.jsonl 2> gpurun_out/t9/flow.err
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -rf -k "driver or local or c5_reduced or bundles" > gpurun_out/t9/pytest.log 2>&1
echo done
