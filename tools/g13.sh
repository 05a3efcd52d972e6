timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/g13_pytest.log 2>&1
JIT=1 timeout 900 python tools/perf_probe.py 2,3,4 > gpurun_out/g13_probe.log 2>&1
timeout 600 python tools/perf_probe.py 3,4 >> gpurun_out/g13_probe.log 2>&1
for cfg in "SMEM_KB=112 RTLSIM_JIT_TPC=2" "SMEM_KB=112 RTLSIM_JIT_TPC=2 LANES=4" "LANES=16"; do
 env JIT=1 $cfg timeout 600 python tools/perf_probe.py 4 >> gpurun_out/g13_probe.log 2>&1
done
