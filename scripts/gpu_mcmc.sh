set -x
timeout 900 python -m pytest tests/test_gpu_mcmc.py -q -x > gpurun_out/pytest_gpu_mcmc.log 2>&1; tail -30 gpurun_out/pytest_gpu_mcmc.log
timeout 300 python scripts/mcmc_time.py m2 > gpurun_out/mcmc_time.log 2>&1; cat gpurun_out/mcmc_time.log
