mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for M in 0 1 2; do
CEC_SUPP_MODE=$M timeout 600 python scripts/time_plan.py c5 3 > gpurun_out/timing_m$M.log 2>&1
CEC_SUPP_MODE=$M timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:supp --csv --log-file gpurun_out/supp_m$M.csv python scripts/time_plan.py c5 1 > /dev/null 2>&1
done
echo done
