# Targeted ncu capture of the tracking kernel (fewer replays than --set full).
set -x
CFG=${CFG:-c3}
TAG=${TAG:-q}
export BENCH_ALLOW_FEW_WARMUP=1
ncu --section SpeedOfLight --section LaunchStats --section Occupancy --section WarpStateStats \
    --section SchedulerStats --section SourceCounters --section MemoryWorkloadAnalysis \
    --section ComputeWorkloadAnalysis --section InstructionStats \
    --clock-control none --import-source on -k regex:track_kernel -s 1 -c 1 \
    -o gpurun_out/prof_${CFG}_${TAG} -f \
    python bench.py --config $CFG --steps 1 --warmup 1 --no-cpu-baseline --no-gather-bench $EXTRA > gpurun_out/prof_bench_${CFG}_${TAG}.log 2>&1
