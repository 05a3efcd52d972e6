export RTLSIM_JIT_CACHE=/tmp/rtlsim_jit_cache
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/g20_pytest.log 2>&1
JIT=1 timeout 900 python tools/perf_probe.py 2,3,4 > gpurun_out/g20_probe.log 2>&1
for cfg in "SMEM_KB=75 RTLSIM_JIT_TMAX=3 RTLSIM_JIT_TPC=3" "SMEM_KB=56 RTLSIM_JIT_TMAX=4 RTLSIM_JIT_TPC=4" "LANES=2 SMEM_KB=75 RTLSIM_JIT_TMAX=3 RTLSIM_JIT_TPC=3"; do
 env JIT=1 $cfg timeout 900 python tools/perf_probe.py 4 >> gpurun_out/g20_probe.log 2>&1
done
for cfg in "RTLSIM_JIT_TMAX=6" "LANES=2 RTLSIM_JIT_TMAX=6" "RTLSIM_JIT_GROUP=1600"; do
 env JIT=1 $cfg timeout 600 python tools/perf_probe.py 3 >> gpurun_out/g20_probe.log 2>&1
done
timeout 900 python bench.py > gpurun_out/g20_bench.log 2>&1
