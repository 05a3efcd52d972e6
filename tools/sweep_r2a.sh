#!/bin/bash
# round-2 sweep: JIT throughput vs op-lanes (L) and tiles per CTA (K)
mkdir -p gpurun_out
python -c "from paper_conf_icpp_linrzkh22_b200 import build; build.build()"
export JIT=1 RTLSIM_JIT_CACHE=/tmp/jc
run() { echo "== $*" ; env "$@" timeout 600 python tools/perf_probe.py $CFG 2>&1 | tail -1; }
CFG=3
for lk in "4 4" "4 2" "2 4" "2 8" "1 4" "1 8" "8 2" "8 4"; do set -- $lk
  run N=65536 LANES=$1 RTLSIM_JIT_TMAX=$2 RTLSIM_JIT_TPC=$2
done
CFG=4
run N=65536 RTLSIM_JIT_OPT=mid
run N=65536 RTLSIM_JIT_OPT=mid LANES=2 SMEM_KB=56 RTLSIM_JIT_TMAX=4 RTLSIM_JIT_TPC=4
run N=65536 RTLSIM_JIT_OPT=mid LANES=1 SMEM_KB=56 RTLSIM_JIT_TMAX=4 RTLSIM_JIT_TPC=4
run N=65536 RTLSIM_JIT_OPT=mid LANES=1 SMEM_KB=28 RTLSIM_JIT_TMAX=8 RTLSIM_JIT_TPC=8
