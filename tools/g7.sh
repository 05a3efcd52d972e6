timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "jit or modes" > gpurun_out/g7_pytest.log 2>&1
for T in 1 2; do for c in 2 3; do JIT=1 RTLSIM_JIT_TPC=$T timeout 300 python tools/perf_probe.py $c >> gpurun_out/g7_probe.log 2>&1; done; done
JIT=1 LANES=16 timeout 900 python tools/perf_probe.py 4 >> gpurun_out/g7_probe.log 2>&1
JIT=1 RTLSIM_JIT_TPC=2 SMEM_KB=110 timeout 900 python tools/perf_probe.py 4 >> gpurun_out/g7_probe.log 2>&1
timeout 900 python tools/ablation.py 3 16384 64 > gpurun_out/g7_ablation3.log 2>&1
