export RTLSIM_JIT_CACHE=/tmp/rtlsim_jit_cache
for v in "RTLSIM_JIT_OPT=mid" "RTLSIM_JIT_OPT=mid RTLSIM_NO_FOLD=1" "RTLSIM_JIT_OPT=mid RTLSIM_JIT_FWD=0" "RTLSIM_JIT_OPT=mid RTLSIM_JIT_GROUP=400" "RTLSIM_JIT_OPT=mid RTLSIM_JIT_FWD=0 RTLSIM_NO_FOLD=1 RTLSIM_JIT_GROUP=400"; do
  env $v timeout 900 python tools/bisect4.py >> gpurun_out/g21_bisect.log 2>&1
done
