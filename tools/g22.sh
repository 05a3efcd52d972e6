export RTLSIM_JIT_CACHE=/tmp/rtlsim_jit_cache
timeout 600 python tools/bisect4.py > gpurun_out/g22_bisect.log 2>&1
timeout 2400 python -m pytest tests -m gpu -x -q > gpurun_out/g22_pytest.log 2>&1
JIT=1 timeout 1200 python tools/perf_probe.py 2,3,4 > gpurun_out/g22_probe.log 2>&1
JIT=1 RTLSIM_JIT_GROUP=1600 timeout 1200 python tools/perf_probe.py 3,4 >> gpurun_out/g22_probe.log 2>&1
timeout 900 python bench.py > gpurun_out/g22_bench.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/g22_smoke.log 2>&1
