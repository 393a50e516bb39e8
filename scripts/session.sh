# The command list of the current gpurun session (overwritten per session; earlier ones are
# in git history).  r02e: GPU suite on the raster-map kernel; default c3/c4 bench lines;
# variant / unique ablations; MCMC line with the algorithmic roofline; ncu captures c3, c4,
# c5 (every 8th seed), NEXT-3 bidirectional + interpolation.
set -x
export TAG=r02e
scripts/gpu.sh test
scripts/gpu.sh bench c3 --steps 5 --warmup 3
scripts/gpu.sh bench c4 --steps 5 --warmup 3
timeout 1500 python scripts/ablations.py --config c3 --reps 1 --only "main,variant instantiation,NEXT-3,NEXT-2" > gpurun_out/r02e_ablations_c3.log 2>&1; tail -9 gpurun_out/r02e_ablations_c3.log
scripts/gpu.sh bench m2 --steps 3 --warmup 3
scripts/gpu.sh ncu c3 track_kernel
scripts/gpu.sh ncu c4 track_kernel
scripts/gpu.sh ncu c5 track_kernel --seed-every 8
TAG=r02e_var scripts/gpu.sh ncu c3 track_kernel --track-flags 6144
