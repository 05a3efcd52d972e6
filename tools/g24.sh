export RTLSIM_JIT_CACHE=/tmp/rtlsim_jit_cache
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/g24_pytest.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/g24_smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/g24_bench.log 2>&1
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/g24_bench_ref.log 2>&1
