# r01f tracking-kernel evidence with the current build: launch list of the bench command and
# one --set full capture of track_kernel (c3), plus the full c3 bench line.
set -x
export BENCH_ALLOW_FEW_WARMUP=1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c3_r01f.csv python bench.py --config c3 --steps 2 --warmup 1 --no-cpu-baseline --no-gather-bench > gpurun_out/launches_bench_c3_r01f.json 2>&1; tail -2 gpurun_out/launches_c3_r01f.csv
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:track_kernel -s 1 -c 1 -o gpurun_out/prof_c3_r01f -f python bench.py --config c3 --steps 1 --warmup 1 --no-cpu-baseline --no-gather-bench > gpurun_out/prof_bench_c3_r01f.log 2>&1; tail -2 gpurun_out/prof_bench_c3_r01f.log
unset BENCH_ALLOW_FEW_WARMUP
timeout 900 python bench.py > gpurun_out/bench_c3_final.json 2> gpurun_out/bench_c3_final.err; cat gpurun_out/bench_c3_final.json
timeout 1500 python bench.py --config c5 --steps 2 --warmup 3 --no-cpu-baseline --emulate-ranks 8 > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err; cut -c1-1500 gpurun_out/bench_c5.json; tail -3 gpurun_out/bench_c5.err
