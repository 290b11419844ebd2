# round 2 (re-entry): larger fuzz campaigns on the final tree (kernels: JIT / AUTO / interpreter;
# the whole flow)
set -x
mkdir -p gpurun_out/r2s2_52
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2s2_52/build.log 2>&1
timeout 1500 python scripts/fuzz_jit.py --engine jit --seeds 1000 --start 10000 > gpurun_out/r2s2_52/fuzz_jit.jsonl 2>&1
timeout 900 python scripts/fuzz_jit.py --engine auto --seeds 1000 --start 20000 > gpurun_out/r2s2_52/fuzz_auto.jsonl 2>&1
timeout 900 python scripts/fuzz_jit.py --engine interp --seeds 1000 --start 30000 > gpurun_out/r2s2_52/fuzz_interp.jsonl 2>&1
timeout 1500 python scripts/fuzz_jit.py --engine auto --miters --seeds 400 --start 40000 --split 65536 > gpurun_out/r2s2_52/fuzz_auto_miters.jsonl 2>&1
timeout 1800 python scripts/fuzz_flow.py --seeds 300 --start 1000 > gpurun_out/r2s2_52/fuzz_flow.jsonl 2>&1
echo done
