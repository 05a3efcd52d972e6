export RTLSIM_JIT_CACHE=/tmp/rtlsim_jit_cache
timeout 600 python tools/bisect4.py > gpurun_out/g23_bisect.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/g23_pytest.log 2>&1
JIT=1 timeout 1200 python tools/perf_probe.py 2,3,4 > gpurun_out/g23_probe.log 2>&1
timeout 900 python bench.py > gpurun_out/g23_bench.log 2>&1
mkdir -p /tmp/rep
JIT=1 timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:rtl_jit -s 64 -c 64 --csv --log-file gpurun_out/g23_cycle_dram.csv python tools/prof_run.py 4 1 3 > gpurun_out/g23_dram.log 2>&1
JIT=1 timeout 900 ncu --set full --clock-control none -k regex:rtl_jit -s 70 -c 1 -o /tmp/rep/c4jit python tools/prof_run.py 4 1 2 > gpurun_out/g23_ncu4.log 2>&1
python tools/ncu_summary.py /tmp/rep/c4jit.ncu-rep gpurun_out/g23_c4jit --stim-cycles 65536 >> gpurun_out/g23_ncu4.log 2>&1
ncu -i /tmp/rep/c4jit.ncu-rep --page raw --csv > gpurun_out/g23_c4jit_raw.csv 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/g23_launches.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/g23_bench_under_ncu.log 2>&1
