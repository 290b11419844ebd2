# round 1c: full GPU suite (incl. full-size C5 golden), default bench (parity vs golden), e2e pipelining sweep
mkdir -p gpurun_out/c7
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c7/build.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu -rf > gpurun_out/c7/pytest.log 2>&1
timeout 600 python bench.py > gpurun_out/c7/bench.log 2>&1
CEC_TIMING=1 timeout 300 python scripts/time_plan.py c5 3 > gpurun_out/c7/time_plan.log 2>&1
timeout 600 python scripts/e2e_sweep.py c5 7 > gpurun_out/c7/e2e_sweep.jsonl 2> gpurun_out/c7/e2e_sweep.err
echo done
