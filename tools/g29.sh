# dead slot-store elimination (RTLSIM_JIT_DSE=1): parity + perf
export RTLSIM_JIT_CACHE=/tmp/rtlsim_jit_cache
export RTLSIM_JIT_DSE=1
JIT=1 timeout 900 python tools/perf_probe.py 3,4 > gpurun_out/g29_probe_dse.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/g29_pytest_dse.log 2>&1
