python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/g3_smoke.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/g3_pytest.log 2>&1
for c in 2 3 4; do timeout 300 python tools/perf_probe.py $c >> gpurun_out/g3_probe.log 2>&1; done
LANES=16 timeout 300 python tools/perf_probe.py 4 >> gpurun_out/g3_probe.log 2>&1
