set -x
mkdir -p gpurun_out
nvidia-smi > gpurun_out/smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/bench_default.log 2>&1
timeout 600 python bench.py --impl reference > gpurun_out/bench_reference.log 2>&1
timeout 900 python scripts/c4_flow.py > gpurun_out/c4_flow.log 2>&1
timeout 3000 python -m pytest tests -m gpu -q -rf > gpurun_out/pytest_gpu.log 2>&1
echo done
