set -x
timeout 900 python -m pytest tests/test_gpu_mcmc.py -q -x > gpurun_out/pytest_gpu_mcmc5.log 2>&1; tail -5 gpurun_out/pytest_gpu_mcmc5.log
for v in vpw1mb4 vpw2mb4 vpw2mb2; do PT_LIB=$PWD/scripts/libpt_mcmc_$v.so timeout 300 python scripts/mcmc_time.py m2 2>&1 | sed "s/^/$v /" | tail -1; done
timeout 300 python scripts/mcmc_time.py m2 2>&1 | sed "s/^/vpw2mb3 /" | tail -1
