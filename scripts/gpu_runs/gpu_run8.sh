set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
B="python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1"
timeout 900 $B --config c3 > gpurun_out/m_c3.log 2>&1
timeout 900 $B > gpurun_out/m_c5.log 2>&1
CEC_NO_SIDE_STREAMS=1 timeout 900 $B > gpurun_out/m_c5_noside.log 2>&1
timeout 300 $B --config c2 > gpurun_out/m_c2.log 2>&1
timeout 300 $B --config c1 > gpurun_out/m_c1.log 2>&1
timeout 3000 python -m pytest tests -m gpu -q -rf > gpurun_out/pytest_gpu.log 2>&1
echo done
