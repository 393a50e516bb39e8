# The command list of the current gpurun session (overwritten per session; earlier ones are
# in git history).  r02g: claim granularity on the DRAM-bound c5 (and c3): whole seeds in
# groups of 32 (default) vs one seed per claim vs seeds split over several CTAs (chunks of
# 2048 / 1024 particles) -- fewer seeds in flight chip-wide = a smaller L2 working set.
set -x
export TAG=r02g
scripts/gpu.sh ab "default env:PT_SEEDS_PER_CLAIM=1 env:PT_CTA_CHUNK=2048 env:PT_CTA_CHUNK=1024" "c5" 1
scripts/gpu.sh ab "default env:PT_SEEDS_PER_CLAIM=1 env:PT_CTA_CHUNK=2048 env:PT_CTA_CHUNK=1024" "c3 c4" 1
