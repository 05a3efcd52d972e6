timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/g15_pytest.log 2>&1
JIT=1 timeout 900 python tools/perf_probe.py 2,3,4 > gpurun_out/g15_probe.log 2>&1
for F in 0 4; do JIT=1 RTLSIM_JIT_FWD=$F timeout 900 python tools/perf_probe.py 3,4 >> gpurun_out/g15_probe.log 2>&1; done
timeout 900 python bench.py > gpurun_out/g15_bench.log 2>&1
