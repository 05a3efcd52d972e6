# forwarding-distance sweep with one function per partition; refreshed ncu evidence
export RTLSIM_JIT_CACHE=/tmp/rtlsim_jit_cache
for f in 4 8; do
  RTLSIM_JIT_FWD=$f JIT=1 timeout 900 python tools/perf_probe.py 3,4 > gpurun_out/g28_probe_fwd$f.log 2>&1
done
mkdir -p /tmp/rep
JIT=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:rtl_jit -s 70 -c 1 -o /tmp/rep/c4jit python tools/prof_run.py 4 1 2 > gpurun_out/g28_ncu4.log 2>&1
python tools/ncu_summary.py /tmp/rep/c4jit.ncu-rep gpurun_out/g28_c4jit --stim-cycles 65536 >> gpurun_out/g28_ncu4.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/g28_launches.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/g28_bench_under_ncu.log 2>&1
