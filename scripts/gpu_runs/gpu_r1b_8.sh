mkdir -p gpurun_out/t8
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/t8/smoke.log 2>&1
timeout 1800 python -m pytest tests -q -m gpu -rf > gpurun_out/t8/pytest_gpu.log 2>&1
timeout 600 python bench.py > gpurun_out/t8/c5.log 2>&1
timeout 900 python bench.py --config c3 --no-cpu-baseline > gpurun_out/t8/c3.log 2>&1
timeout 300 python bench.py --config c2 --no-cpu-baseline > gpurun_out/t8/c2.log 2>&1
timeout 300 python bench.py --config c2bug --no-cpu-baseline > gpurun_out/t8/c2bug.log 2>&1
timeout 300 python bench.py --config c1 --no-cpu-baseline > gpurun_out/t8/c1.log 2>&1
timeout 600 python scripts/c4_flow.py > gpurun_out/t8/c4_flow.jsonl 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/t8/c3_launches.csv python bench.py --config c3 --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1
echo done
