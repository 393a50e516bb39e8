set -x
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_full.log 2>&1; tail -3 gpurun_out/pytest_gpu_full.log
timeout 600 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err; tail -2 gpurun_out/bench_full.err; cat gpurun_out/bench_full.json
timeout 600 python bench.py --config c4 --no-cpu-baseline > gpurun_out/bench_c4.json 2>&1
CFG=c3 TAG=r01e timeout 1500 bash scripts/profile_quick.sh
export BENCH_ALLOW_FEW_WARMUP=1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c3_r01e.csv python bench.py --config c3 --steps 2 --warmup 1 --no-cpu-baseline --no-gather-bench > /dev/null 2>&1
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,gpu__time_duration.sum --clock-control none -k regex:track_kernel -s 1 -c 1 --csv --log-file gpurun_out/dram_c3_r01e.csv python bench.py --config c3 --steps 1 --warmup 1 --no-cpu-baseline --no-gather-bench > /dev/null 2>&1
