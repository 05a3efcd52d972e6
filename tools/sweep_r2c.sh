#!/bin/bash
# round-2 sweep c: aligned step barrier + op-lane affinity; op-lane counts
mkdir -p gpurun_out
python -c "from paper_conf_icpp_linrzkh22_b200 import build; build.build()"
export JIT=1 RTLSIM_JIT_CACHE=/tmp/jc
run() { echo "== $*" ; env "$@" timeout 900 python tools/perf_probe.py $CFG 2>&1 | tail -1; }
CFG=3
run N=65536 LANES=4 RTLSIM_JIT_TMAX=4 RTLSIM_JIT_TPC=4
run N=65536 LANES=8 RTLSIM_JIT_TMAX=4 RTLSIM_JIT_TPC=4
run N=65536 LANES=8 RTLSIM_JIT_TMAX=4 RTLSIM_JIT_TPC=4 RTLSIM_AFFINITY=0
run N=65536 LANES=16 RTLSIM_JIT_TMAX=2 RTLSIM_JIT_TPC=2
CFG=4
run N=65536 RTLSIM_JIT_OPT=mid LANES=8 RTLSIM_JIT_TMAX=2 RTLSIM_JIT_TPC=2
run N=65536 RTLSIM_JIT_OPT=mid LANES=8 RTLSIM_JIT_TMAX=2 RTLSIM_JIT_TPC=2 RTLSIM_AFFINITY=0
run N=65536 RTLSIM_JIT_OPT=mid LANES=16 RTLSIM_JIT_TMAX=2 RTLSIM_JIT_TPC=2
run N=65536 LANES=8 RTLSIM_JIT_TMAX=2 RTLSIM_JIT_TPC=2
