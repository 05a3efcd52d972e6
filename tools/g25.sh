export RTLSIM_JIT_CACHE=/tmp/rtlsim_jit_cache
for v in "" "RTLSIM_OLD_COST=1"; do
  env $v JIT=1 timeout 1200 python tools/perf_probe.py 3,4 >> gpurun_out/g25_probe.log 2>&1
done
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -k "jit or full" > gpurun_out/g25_pytest.log 2>&1
