# round 1c: C3 device-step sweep: side streams and bundle threshold
mkdir -p gpurun_out/c22
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c22/build.log 2>&1
run() { timeout 600 python bench.py --no-cpu-baseline --config c3 --steps 5 --e2e-steps 1 > gpurun_out/c22/$1.log 2>&1; }
run base
CEC_SIDE_STREAMS=8 run ss8
CEC_SIDE_STREAMS=16 run ss16
CEC_BUNDLE_BELOW=8589934592 run bb33
CEC_BUNDLE_BELOW=34359738368 run bb35
CEC_BUNDLE_BELOW=68719476736 run bb36
echo done
