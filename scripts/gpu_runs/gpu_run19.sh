set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 python scripts/profile_groups.py c3 > gpurun_out/groups_c3.log 2>&1
timeout 600 python scripts/profile_groups.py c5 > gpurun_out/groups_c5.log 2>&1
timeout 600 python bench.py --config c2 --no-cpu-baseline > gpurun_out/bench_c2.log 2>&1
echo done
