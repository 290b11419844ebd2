# round 1c: host phase timings of the C3 / C5 public call, scaling projection refresh
mkdir -p gpurun_out/c18
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c18/build.log 2>&1
CEC_TIMING=1 timeout 300 python scripts/time_plan.py c3 3 > gpurun_out/c18/time_plan_c3.log 2>&1
CEC_TIMING=1 timeout 300 python scripts/time_plan.py c5 3 > gpurun_out/c18/time_plan_c5.log 2>&1
timeout 900 python scripts/scale_emulate.py > gpurun_out/c18/scale.jsonl 2> gpurun_out/c18/scale.err
echo done
