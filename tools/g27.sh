# one JIT function per partition (no R2UR per access) + N-specialised windows
export RTLSIM_JIT_CACHE=/tmp/rtlsim_jit_cache
JIT=1 timeout 900 python tools/perf_probe.py 3,4 > gpurun_out/g27_probe.log 2>&1
timeout 900 python bench.py > gpurun_out/g27_bench.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/g27_pytest.log 2>&1
