#!/bin/bash
# round-2 sweep d: config 4 occupancy vs shared-memory budget (ptxas -O3)
mkdir -p gpurun_out
python -c "from paper_conf_icpp_linrzkh22_b200 import build; build.build()"
export JIT=1 RTLSIM_JIT_CACHE=/tmp/jc
run() { echo "== $*" ; env "$@" timeout 1200 python tools/perf_probe.py $CFG 2>&1 | tail -1; }
CFG=4
run N=65536 LANES=8 RTLSIM_JIT_TMAX=4 RTLSIM_JIT_TPC=4 SMEM_KB=56
run N=65536 LANES=16 RTLSIM_JIT_TMAX=2 RTLSIM_JIT_TPC=2
run N=65536 LANES=4 RTLSIM_JIT_TMAX=4 RTLSIM_JIT_TPC=4 SMEM_KB=56
run N=65536 LANES=8 RTLSIM_JIT_TMAX=2 RTLSIM_JIT_TPC=2 RTLSIM_JIT_FWD=4
