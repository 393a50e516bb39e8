set -x
timeout 900 python -m pytest tests/test_gpu_mcmc.py -q -x > gpurun_out/pytest_gpu_mcmc3.log 2>&1; tail -5 gpurun_out/pytest_gpu_mcmc3.log
for v in fma0 mb3; do PT_LIB=$PWD/scripts/libpt_mcmc_$v.so timeout 300 python scripts/mcmc_time.py m2 2>&1 | sed "s/^/$v /" | tail -1; done
timeout 300 python scripts/mcmc_time.py m2 2>&1 | sed "s/^/default /" | tail -1
timeout 1500 python scripts/ablations.py --config c3 --reps 1 > gpurun_out/ablations_c3.log 2>&1; tail -16 gpurun_out/ablations_c3.log
