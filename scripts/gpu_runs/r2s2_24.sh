# round 2 (re-entry): fuzz campaigns on the current tree: AUTO engine (interpreter windows skip the
# id-order evaluation), the public call with large-windows-first splits, JIT miters
set -x
mkdir -p gpurun_out/r2s2_24
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2s2_24/build.log 2>&1
timeout 900 python scripts/fuzz_jit.py --engine auto --seeds 400 > gpurun_out/r2s2_24/fuzz_auto.jsonl 2>&1
timeout 900 python scripts/fuzz_jit.py --engine auto --seeds 300 --start 400 --split 65536 > gpurun_out/r2s2_24/fuzz_auto_split.jsonl 2>&1
timeout 900 python scripts/fuzz_jit.py --engine auto --miters --seeds 200 --start 700 --split 1048576 > gpurun_out/r2s2_24/fuzz_auto_miters_split.jsonl 2>&1
timeout 900 python scripts/fuzz_jit.py --engine jit --miters --seeds 200 --start 900 > gpurun_out/r2s2_24/fuzz_jit_miters.jsonl 2>&1
echo done
