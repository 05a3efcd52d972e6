V4=1 timeout 600 python tools/perf_probe.py 3,4 > gpurun_out/g12_probe_v4.log 2>&1
mkdir -p /tmp/rep
V4=1 PROF_N=8192 timeout 900 ncu --set full --import-source on --clock-control none -k regex:rtl_eval_v4 -s 2 -c 1 -o /tmp/rep/c4v4 python tools/prof_run.py 4 1 3 > gpurun_out/g12_ncu4.log 2>&1
python tools/ncu_summary.py /tmp/rep/c4v4.ncu-rep gpurun_out/g12_c4v4 --stim-cycles 8192 >> gpurun_out/g12_ncu4.log 2>&1
ncu -i /tmp/rep/c4v4.ncu-rep --page raw --csv > gpurun_out/g12_c4v4_raw.csv 2>&1
ncu -i /tmp/rep/c4v4.ncu-rep --page source --csv --print-source sass > gpurun_out/g12_c4v4_src.csv 2>&1
ls -la /tmp/rep gpurun_out >> gpurun_out/g12_ncu4.log
