# The command list of the current gpurun session (overwritten per session; earlier ones are
# in git history).  r02h: c5 seeds-per-claim sweep (whole seeds per CTA claim: 1, 4, 8, 32),
# interleaved x2 (r02g: 1 seed per claim 94.4 G vs 88.6 G default, but at different clocks).
set -x
export TAG=r02h
scripts/gpu.sh ab "env:PT_SEEDS_PER_CLAIM=1 env:PT_SEEDS_PER_CLAIM=4 env:PT_SEEDS_PER_CLAIM=8 default" "c5" 2
