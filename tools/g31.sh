export RTLSIM_JIT_CACHE=/tmp/rtlsim_jit_cache
timeout 600 python -m pytest tests/test_gpu_parity.py -q -k "rebind or jit_sequential or jit_lanes" > gpurun_out/g31_pytest.log 2>&1
