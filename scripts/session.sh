# The command list of the current gpurun session (overwritten per session; earlier ones are
# in git history).  r02i: keep the map in L2 -- map REDs with an L2 evict_last policy (redel)
# and the map as a persisting access-policy window (env PT_MAP_PERSIST) vs the default, on
# c3 / c4 and c5 (c5 now claims 4 seeds at a time: record volume > 4 GB).
set -x
export TAG=r02i
scripts/gpu.sh ab "default redel env:PT_MAP_PERSIST=1" "c3 c4" 2
scripts/gpu.sh ab "default redel env:PT_MAP_PERSIST=1" "c5" 1
