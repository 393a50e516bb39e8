# The command list of the current gpurun session (overwritten per session; earlier ones are
# in git history).  r02f: the deferred unique-map probe (GPU tests + ablation line); L2 fetch
# granularity A/B (cudaLimitMaxL2FetchGranularity 32 / 64 B vs the driver default) on c3, c4
# and c5 (every 4th seed).
set -x
export TAG=r02f
timeout 1200 python -m pytest tests -m gpu -x -q -k "unique or smoke or multirank or sanitizer" > gpurun_out/r02f_pytest_unique.log 2>&1; tail -3 gpurun_out/r02f_pytest_unique.log
timeout 900 python scripts/ablations.py --config c3 --reps 1 --only "main,NEXT-2" > gpurun_out/r02f_ablations_c3.log 2>&1; tail -4 gpurun_out/r02f_ablations_c3.log
scripts/gpu.sh ab "default l2f32 l2f64" "c3 c4" 2
scripts/gpu.sh ab "default l2f32 l2f64" "c5" 1 --seed-every 4
