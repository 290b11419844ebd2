set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 1200 python -m pytest tests -m gpu -q -rf -k "cut or driver" > gpurun_out/pytest_cuts.log 2>&1
timeout 900 python scripts/c4_flow.py > gpurun_out/c4_flow.log 2>&1
CEC_CUTS_HOST=1 timeout 900 python scripts/c4_flow.py > gpurun_out/c4_flow_hostcuts.log 2>&1
echo done
