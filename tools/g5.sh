timeout 600 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/g5_pytest.log 2>&1
for c in 2 3 4; do timeout 300 python tools/perf_probe.py $c >> gpurun_out/g5_probe.log 2>&1; done
LANES=8 timeout 300 python tools/perf_probe.py 3 >> gpurun_out/g5_probe.log 2>&1
LANES=8 timeout 300 python tools/perf_probe.py 4 >> gpurun_out/g5_probe.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:rtl_eval_v4 -s 2 -c 1 -o gpurun_out/g5_c3 python tools/prof_run.py 3 4 3 > gpurun_out/g5_ncu3.log 2>&1
