# ncu evidence for the tracking kernel (one GPU): launch list + one --set full capture.
set -x
CFG=${CFG:-c3}
TAG=${TAG:-r01}
export BENCH_ALLOW_FEW_WARMUP=1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${CFG}_${TAG}.csv \
    python bench.py --config $CFG --steps 2 --warmup 1 --no-cpu-baseline --no-gather-bench > gpurun_out/launches_bench_${CFG}_${TAG}.json 2>&1
ncu --set full --clock-control none --import-source on -k regex:"track_(spec_)?kernel" -s 1 -c 1 \
    -o gpurun_out/prof_${CFG}_${TAG} -f \
    python bench.py --config $CFG --steps 1 --warmup 1 --no-cpu-baseline --no-gather-bench > gpurun_out/prof_bench_${CFG}_${TAG}.log 2>&1
ls -la gpurun_out
