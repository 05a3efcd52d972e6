set -x
for L in 4 8 16; do for S in 0 110 72; do
 JIT=1 LANES=$L SMEM_KB=$S timeout 300 python tools/perf_probe.py 3 >> gpurun_out/g2_probe.log 2>&1
done; done
JIT=1 LANES=8 timeout 600 ncu --set full --clock-control none --import-source on -k regex:rtl_jit -s 8 -c 1 -o gpurun_out/g2_c3_jit python tools/prof_run.py 3 4 3 > gpurun_out/g2_ncu.log 2>&1
JIT=1 SMEM_KB=110 timeout 900 python tools/perf_probe.py 4 >> gpurun_out/g2_probe.log 2>&1
