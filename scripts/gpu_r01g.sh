# r01g evidence with the bricked record layout (default PT_BRICK=4): GPU suite, smoke,
# default bench line (c3), c4 line, launch list + one --set full capture of track_kernel.
set -x
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r01g_pytest_gpu.log 2>&1; tail -3 gpurun_out/r01g_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r01g_smoke.log 2>&1; tail -1 gpurun_out/r01g_smoke.log
timeout 900 python bench.py > gpurun_out/r01g_bench_c3.json 2> gpurun_out/r01g_bench_c3.err; cut -c1-300 gpurun_out/r01g_bench_c3.json
timeout 900 python bench.py --config c4 --no-cpu-baseline > gpurun_out/r01g_bench_c4.json 2> gpurun_out/r01g_bench_c4.err; cut -c1-300 gpurun_out/r01g_bench_c4.json
export BENCH_ALLOW_FEW_WARMUP=1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r01g_launches_c3.csv python bench.py --config c3 --steps 2 --warmup 1 --no-cpu-baseline --no-gather-bench > gpurun_out/r01g_launches_bench_c3.json 2>&1; tail -2 gpurun_out/r01g_launches_c3.csv
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:track_kernel -s 1 -c 1 -o gpurun_out/r01g_prof_c3 -f python bench.py --config c3 --steps 1 --warmup 1 --no-cpu-baseline --no-gather-bench > gpurun_out/r01g_prof_bench_c3.log 2>&1; tail -2 gpurun_out/r01g_prof_bench_c3.log
