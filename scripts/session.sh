# The command list of the current gpurun session (overwritten per session; earlier ones are
# in git history).  r02c: GPU suite on the compile-time-variant kernels and the record-ordered
# map; variant / unique ablations; tile A/B; default c3 bench line.
set -x
export TAG=r02c
scripts/gpu.sh test
timeout 1500 python scripts/ablations.py --config c3 --reps 1 --only "main,variant instantiation,NEXT-3,NEXT-2" > gpurun_out/r02c_ablations_c3.log 2>&1; tail -9 gpurun_out/r02c_ablations_c3.log
scripts/gpu.sh ab "default tile" "c3 c4" 2
scripts/gpu.sh bench c3 --steps 5 --warmup 3
