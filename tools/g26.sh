# windowed (N-specialised) JIT addressing: A/B, parity, bench
export RTLSIM_JIT_CACHE=/tmp/rtlsim_jit_cache
JIT=1 timeout 900 python tools/perf_probe.py 3,4 > gpurun_out/g26_probe.log 2>&1
RTLSIM_JIT_GENERIC=1 JIT=1 timeout 900 python tools/perf_probe.py 3,4 > gpurun_out/g26_probe_generic.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/g26_pytest.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/g26_smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/g26_bench.log 2>&1
