nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/g9_smi.txt; nproc >> gpurun_out/g9_smi.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/g9_smoke.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/g9_pytest.log 2>&1
JIT=1 timeout 900 python tools/perf_probe.py 2,3,4 > gpurun_out/g9_probe_jit.log 2>&1
timeout 600 python tools/perf_probe.py 2,3,4 > gpurun_out/g9_probe_interp.log 2>&1
timeout 900 python bench.py > gpurun_out/g9_bench.log 2>&1
