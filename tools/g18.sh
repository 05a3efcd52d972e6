timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "mcmc" > gpurun_out/g18_pytest.log 2>&1
timeout 1200 python tools/mcmc_partition.py 3 4 24 16384 4 > gpurun_out/g18_mcmc3.log 2>&1
timeout 1500 python tools/mcmc_partition.py 4 32 8 8192 2 > gpurun_out/g18_mcmc4.log 2>&1
timeout 900 python tools/ablation.py 3 16384 64 > gpurun_out/g18_ablation3.log 2>&1
