mkdir -p /tmp/rep
# launch list of the bench command (cold-cache, serialised: shares only)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/g17_launches.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/g17_bench_under_ncu.log 2>&1
# DRAM bytes of every partition kernel of one cycle at the bench size (N=65536)
JIT=1 timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:rtl_jit -s 64 -c 64 --csv --log-file gpurun_out/g17_cycle_dram.csv python tools/prof_run.py 4 1 3 > gpurun_out/g17_dram.log 2>&1
# full set on one partition kernel (N=65536)
JIT=1 timeout 900 ncu --set full --clock-control none -k regex:rtl_jit -s 70 -c 1 -o /tmp/rep/c4jit python tools/prof_run.py 4 1 2 > gpurun_out/g17_ncu4.log 2>&1
python tools/ncu_summary.py /tmp/rep/c4jit.ncu-rep gpurun_out/g17_c4jit --stim-cycles 65536 >> gpurun_out/g17_ncu4.log 2>&1
ncu -i /tmp/rep/c4jit.ncu-rep --page raw --csv > gpurun_out/g17_c4jit_raw.csv 2>&1
JIT=1 timeout 600 ncu --set full --clock-control none -k regex:rtl_jit -s 10 -c 1 -o /tmp/rep/c3jit python tools/prof_run.py 3 2 2 > gpurun_out/g17_ncu3.log 2>&1
python tools/ncu_summary.py /tmp/rep/c3jit.ncu-rep gpurun_out/g17_c3jit --stim-cycles 16384 >> gpurun_out/g17_ncu3.log 2>&1
