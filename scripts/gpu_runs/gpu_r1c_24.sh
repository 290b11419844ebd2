# round 1c: cooperative single-launch level loops (classes, reduce): block shape sweep vs per-level launches
mkdir -p gpurun_out/c24
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c24/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_reduce.py tests/test_gpu_classes.py -q -m gpu -rf > gpurun_out/c24/pytest.log 2>&1
CEC_RS_LEVEL_LAUNCHES=1 CEC_RD_BATCH_LAUNCHES=1 timeout 600 python scripts/bench_flow.py > gpurun_out/c24/levels.log 2>&1
CEC_COOP_T=256 CEC_COOP_BPS=8 timeout 600 python scripts/bench_flow.py > gpurun_out/c24/t256b8.log 2>&1
CEC_COOP_T=1024 CEC_COOP_BPS=1 timeout 600 python scripts/bench_flow.py > gpurun_out/c24/t1024b1.log 2>&1
CEC_COOP_T=512 CEC_COOP_BPS=1 timeout 600 python scripts/bench_flow.py > gpurun_out/c24/t512b1.log 2>&1
CEC_COOP_T=256 CEC_COOP_BPS=2 timeout 600 python scripts/bench_flow.py > gpurun_out/c24/t256b2.log 2>&1
echo done
