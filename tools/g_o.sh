#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/o_build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_tmem.py -q > gpurun_out/o_pytest_tmem.log 2>&1; echo "pytest rc=$?" >> gpurun_out/o_pytest_tmem.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -k "config4 or config5" > gpurun_out/o_pytest_full.log 2>&1; echo "pytest rc=$?" >> gpurun_out/o_pytest_full.log
timeout 900 python bench.py > gpurun_out/o_bench.log 2>&1
