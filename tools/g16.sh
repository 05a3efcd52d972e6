timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/g16_pytest.log 2>&1
JIT=1 timeout 900 python tools/perf_probe.py 2,3,4 > gpurun_out/g16_probe.log 2>&1
