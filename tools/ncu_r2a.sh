#!/bin/bash
# round-2: ncu of one config-3 partition kernel under several (L, K) shapes
mkdir -p gpurun_out
python -c "from paper_conf_icpp_linrzkh22_b200 import build; build.build()"
export JIT=1 PROF_N=65536 RTLSIM_JIT_CACHE=/tmp/jc
prof() { tag=$1; shift; env "$@" timeout 900 ncu --set full --import-source on --clock-control none -k regex:rtl_jit_part -s 19 -c 1 -o gpurun_out/r2a_$tag -f python tools/prof_run.py 3 2 2 > gpurun_out/r2a_$tag.log 2>&1; echo "$tag rc=$?"; }
prof l4k2 LANES=4 RTLSIM_JIT_TMAX=2 RTLSIM_JIT_TPC=2
prof l4k4 LANES=4 RTLSIM_JIT_TMAX=4 RTLSIM_JIT_TPC=4
prof l8k4 LANES=8 RTLSIM_JIT_TMAX=4 RTLSIM_JIT_TPC=4
prof l1k4 LANES=1 RTLSIM_JIT_TMAX=4 RTLSIM_JIT_TPC=4
