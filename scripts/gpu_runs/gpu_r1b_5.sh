mkdir -p gpurun_out/t5
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/t5/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_reduce.py tests/test_gpu_classes.py -q -m gpu -rf > gpurun_out/t5/pytest_new.log 2>&1
timeout 1200 python scripts/bench_flow.py --configs c2,c3,c5 > gpurun_out/t5/flow.jsonl 2> gpurun_out/t5/flow.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/t5/flow_launches.csv python scripts/bench_flow.py --configs c5 --reps 1 --no-oracle > /dev/null 2>&1
echo done
