mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
CEC_SUPP_MODE=3 timeout 600 python -m pytest tests -q -m gpu -x -k "supports or pipelined or c5_full" > gpurun_out/test_gpu.log 2>&1
for M in 3; do
CEC_SUPP_MODE=$M timeout 600 python scripts/time_plan.py c5 3 > gpurun_out/timing_m$M.log 2>&1
CEC_SUPP_MODE=$M timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:supp --csv --log-file gpurun_out/supp_m$M.csv python scripts/time_plan.py c5 1 > /dev/null 2>&1
done
echo done
