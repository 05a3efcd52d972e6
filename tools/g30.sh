# final: DSE on by default — smoke, bench, reference arm, parity subset
export RTLSIM_JIT_CACHE=/tmp/rtlsim_jit_cache
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/g30_smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/g30_bench.log 2>&1
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/g30_bench_ref.log 2>&1
timeout 900 python -m pytest tests/test_gpu_fullsize.py tests/test_gpu_parity.py -q -x -k "jit or full" > gpurun_out/g30_pytest.log 2>&1
