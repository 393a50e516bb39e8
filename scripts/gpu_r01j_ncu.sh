# r01j: one ncu --set full capture of the tracking kernel (6-step rounds), c3
set -x
export BENCH_ALLOW_FEW_WARMUP=1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"track_kernel" -s 1 -c 1 \
    -o gpurun_out/prof_c3_r01j -f \
    python bench.py --config c3 --steps 1 --warmup 1 --no-cpu-baseline --no-gather-bench > gpurun_out/prof_bench_c3_r01j.log 2>&1
ls -la gpurun_out
