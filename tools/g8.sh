JIT=1 PROF_N=8192 timeout 900 ncu --set full --clock-control none --import-source on -k regex:rtl_jit -s 70 -c 1 -o gpurun_out/g8_c4jit python tools/prof_run.py 4 1 2 > gpurun_out/g8_ncu4.log 2>&1
JIT=1 RTLSIM_JIT_TPC=2 timeout 600 ncu --set full --clock-control none --import-source on -k regex:rtl_jit -s 10 -c 1 -o gpurun_out/g8_c3jit python tools/prof_run.py 3 2 2 > gpurun_out/g8_ncu3.log 2>&1
