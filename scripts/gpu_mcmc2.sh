set -x
timeout 600 python bench.py --config m2 --steps 3 --warmup 3 > gpurun_out/bench_m2.json 2> gpurun_out/bench_m2.err; tail -3 gpurun_out/bench_m2.err; cat gpurun_out/bench_m2.json
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mcmc_kernel -c 1 -o gpurun_out/prof_mcmc_m2 -f python bench.py --config m2 --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/prof_mcmc_m2.log 2>&1; tail -3 gpurun_out/prof_mcmc_m2.log
