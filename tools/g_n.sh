#!/bin/bash
# TMEM mode (RTLSIM_JIT_TMEM=1): parity subset + perf on configs 3/4
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/n_build.log 2>&1
export RTLSIM_JIT_TMEM=1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "jit_tiny or jit_comb or jit_sequential or jit_rebind or jit_m1 or jit_dag or shaped_reduced or no_dce or jit_lanes" > gpurun_out/n_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/n_pytest.log
export JIT=1 RTLSIM_JIT_CACHE=/tmp/jc N=65536
run() { echo "== $*" ; env "$@" timeout 600 python tools/perf_probe.py $CFG 2>&1 | tail -2; }
( CFG=3; run RTLSIM_JIT_TMEM=1; run RTLSIM_JIT_TMEM=0; CFG=4; run RTLSIM_JIT_TMEM=1 ) > gpurun_out/n_probe.log 2>&1
