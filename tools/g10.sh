timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k smem > gpurun_out/g10_pytest.log 2>&1
for cfg in "SMEM_KB=110 RTLSIM_JIT_TPC=2" "SMEM_KB=72 RTLSIM_JIT_TPC=3" "LANES=16" "LANES=4"; do
 env JIT=1 $cfg timeout 600 python tools/perf_probe.py 4 >> gpurun_out/g10_probe4.log 2>&1
done
JIT=1 PROF_N=8192 timeout 900 ncu --set full --clock-control none --import-source on -k regex:rtl_jit -s 70 -c 1 -o gpurun_out/g10_c4jit python tools/prof_run.py 4 1 2 > gpurun_out/g10_ncu4.log 2>&1
JIT=1 timeout 600 ncu --set full --clock-control none --import-source on -k regex:rtl_jit -s 10 -c 1 -o gpurun_out/g10_c3jit python tools/prof_run.py 3 2 2 > gpurun_out/g10_ncu3.log 2>&1
