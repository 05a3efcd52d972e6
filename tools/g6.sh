timeout 600 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/g6_pytest.log 2>&1
for L in 8 16; do for c in 2 3 4; do LANES=$L timeout 300 python tools/perf_probe.py $c >> gpurun_out/g6_probe.log 2>&1; done; done
LANES=8 timeout 600 ncu --set full --clock-control none --import-source on -k regex:rtl_eval_v4 -s 2 -c 1 -o gpurun_out/g6_c3 python tools/prof_run.py 3 4 3 > gpurun_out/g6_ncu3.log 2>&1
LANES=8 PROF_N=8192 timeout 900 ncu --set full --clock-control none --import-source on -k regex:rtl_eval_v4 -s 2 -c 1 -o gpurun_out/g6_c4 python tools/prof_run.py 4 1 3 > gpurun_out/g6_ncu4.log 2>&1
