export RTLSIM_JIT_CACHE=/tmp/rtlsim_jit_cache
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/g19_pytest.log 2>&1
JIT=1 timeout 900 python tools/perf_probe.py 2,3,4 > gpurun_out/g19_probe.log 2>&1
JIT=1 RTLSIM_JIT_OPT=O3 timeout 1200 python tools/perf_probe.py 3,4 >> gpurun_out/g19_probe.log 2>&1
JIT=1 RTLSIM_JIT_GROUP=800 timeout 1200 python tools/perf_probe.py 3,4 >> gpurun_out/g19_probe.log 2>&1
timeout 900 python bench.py > gpurun_out/g19_bench.log 2>&1
