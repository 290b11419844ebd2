# round 1c: C3 e2e with pipelined planning forced (CEC_PIPELINE=4) and schedule variants
mkdir -p gpurun_out/c21
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c21/build.log 2>&1
timeout 600 python bench.py --no-cpu-baseline --config c3 --steps 3 --e2e-steps 5 > gpurun_out/c21/c3_base.log 2>&1
CEC_PIPELINE=4 timeout 600 python bench.py --no-cpu-baseline --config c3 --steps 3 --e2e-steps 5 > gpurun_out/c21/c3_pipe.log 2>&1
CEC_PIPELINE=4 CEC_PIPE_FIRST=0.1 CEC_PIPE_GROWTH=2 timeout 600 python bench.py --no-cpu-baseline --config c3 --steps 3 --e2e-steps 5 > gpurun_out/c21/c3_pipe10.log 2>&1
CEC_PIPELINE=4 CEC_PIPE_FIRST=0.25 CEC_PIPE_GROWTH=1.5 timeout 600 python bench.py --no-cpu-baseline --config c3 --steps 3 --e2e-steps 5 > gpurun_out/c21/c3_pipe25.log 2>&1
echo done
