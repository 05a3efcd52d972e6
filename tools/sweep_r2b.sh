#!/bin/bash
# round-2 sweep b: per-tile named barriers (RTLSIM_JIT_TBAR) and op-lane counts
mkdir -p gpurun_out
python -c "from paper_conf_icpp_linrzkh22_b200 import build; build.build()"
export JIT=1 RTLSIM_JIT_CACHE=/tmp/jc
run() { echo "== $*" ; env "$@" timeout 900 python tools/perf_probe.py $CFG 2>&1 | tail -1; }
CFG=3
run N=65536 LANES=4 RTLSIM_JIT_TMAX=4 RTLSIM_JIT_TPC=4 RTLSIM_JIT_TBAR=1
run N=65536 LANES=8 RTLSIM_JIT_TMAX=4 RTLSIM_JIT_TPC=4 RTLSIM_JIT_TBAR=1
run N=65536 LANES=1 RTLSIM_JIT_TMAX=4 RTLSIM_JIT_TPC=4 RTLSIM_JIT_TBAR=1
run N=65536 LANES=1 RTLSIM_JIT_TMAX=8 RTLSIM_JIT_TPC=4 RTLSIM_JIT_TBAR=1 SMEM_KB=28
CFG=4
run N=65536 RTLSIM_JIT_OPT=mid LANES=8 RTLSIM_JIT_TMAX=2 RTLSIM_JIT_TPC=2
run N=65536 RTLSIM_JIT_OPT=mid LANES=8 RTLSIM_JIT_TMAX=2 RTLSIM_JIT_TPC=2 RTLSIM_JIT_TBAR=1
run N=65536 RTLSIM_JIT_OPT=mid LANES=4 RTLSIM_JIT_TBAR=1
