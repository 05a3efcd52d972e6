# config-4 sweep: op-lanes x tiles per CTA x smem budget (JIT)
for cfg in "LANES=4 SMEM_KB=112 RTLSIM_JIT_TMAX=2 RTLSIM_JIT_TPC=2" "LANES=2 SMEM_KB=112 RTLSIM_JIT_TMAX=2 RTLSIM_JIT_TPC=2" \
           "LANES=2 SMEM_KB=75 RTLSIM_JIT_TMAX=3 RTLSIM_JIT_TPC=3" "LANES=4 SMEM_KB=75 RTLSIM_JIT_TMAX=3 RTLSIM_JIT_TPC=3" \
           "LANES=1 SMEM_KB=56 RTLSIM_JIT_TMAX=4 RTLSIM_JIT_TPC=4" "LANES=2 SMEM_KB=56 RTLSIM_JIT_TMAX=4 RTLSIM_JIT_TPC=4"; do
 env JIT=1 $cfg timeout 600 python tools/perf_probe.py 4 >> gpurun_out/g14_probe4.log 2>&1
done
for cfg in "LANES=8 RTLSIM_JIT_TMAX=2" "LANES=4 RTLSIM_JIT_TMAX=4" "LANES=2 RTLSIM_JIT_TMAX=5" "LANES=4 RTLSIM_JIT_TMAX=5" "LANES=1 RTLSIM_JIT_TMAX=5"; do
 env JIT=1 $cfg timeout 600 python tools/perf_probe.py 3 >> gpurun_out/g14_probe3.log 2>&1
done
for cfg in "LANES=8 RTLSIM_JIT_TMAX=2" "LANES=4 RTLSIM_JIT_TMAX=4" "LANES=2 RTLSIM_JIT_TMAX=4"; do
 env JIT=1 $cfg timeout 600 python tools/perf_probe.py 2 >> gpurun_out/g14_probe2.log 2>&1
done
