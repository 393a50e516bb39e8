#!/usr/bin/env bash
# One parameterised driver for the GPU-side experiments (run under gpurun from the repo root).
#   scripts/gpu.sh test [pytest -k expr]     GPU suite (+ smoke) -> gpurun_out/${TAG}_pytest_gpu.log
#   scripts/gpu.sh bench CFG [bench args]    one bench.py line   -> gpurun_out/${TAG}_bench_${CFG}.json
#   scripts/gpu.sh ab "LIBS" "CFGS" REPS     interleaved same-box A/B of experiment builds
#                                            (LIBS: default, names of scripts/libpt_<name>.so
#                                            built with scripts/build_variant.py, or
#                                            env:VAR=v,VAR2=w = the default build under that env)
#   scripts/gpu.sh ncu CFG [KREGEX] [args]   launch list (gpu__time_duration) + one --set full capture
# TAG (env, default r02) prefixes every output file.
set -u
TAG=${TAG:-r02}
mkdir -p gpurun_out
cmd=${1:-}; shift || true
case "$cmd" in
test)
    K=${1:-}
    timeout 2400 python -m pytest tests -m gpu -x -q ${K:+-k "$K"} > gpurun_out/${TAG}_pytest_gpu.log 2>&1
    tail -5 gpurun_out/${TAG}_pytest_gpu.log
    timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1
    tail -2 gpurun_out/${TAG}_smoke.log ;;
bench)
    CFG=$1; shift
    timeout 1200 python bench.py --config $CFG "$@" > gpurun_out/${TAG}_bench_${CFG}.json 2> gpurun_out/${TAG}_bench_${CFG}.err
    cut -c1-600 gpurun_out/${TAG}_bench_${CFG}.json; tail -3 gpurun_out/${TAG}_bench_${CFG}.err ;;
ab)
    LIBS=$1; CFGS=$2; REPS=${3:-2}; shift 3 || true
    for rep in $(seq $REPS); do for lib in $LIBS; do for cfg in $CFGS; do
        ENVS=""
        if [ "$lib" = default ]; then L=$PWD/paper_conf_ipps_xuzwrwxgxy12_b200/libpt.so
        elif [[ "$lib" == env:* ]]; then L=$PWD/paper_conf_ipps_xuzwrwxgxy12_b200/libpt.so; ENVS=${lib#env:}; ENVS=${ENVS//,/ }
        else L=$PWD/scripts/libpt_$lib.so; fi
        env $ENVS PT_LIB=$L timeout 900 python bench.py --config $cfg --steps 3 --warmup 3 --no-cpu-baseline --no-gather-bench \
            --no-parity --no-lengths --no-e2e "$@" 2>/dev/null | tail -1 | python -c "
import json, sys
d = json.loads(sys.stdin.read())
print('$lib', '$cfg', round(d['value'] / 1e9, 6), 'G', d['unit'], round(d['roofline'].get('kernel_ms', 0.0), 2), 'ms',
      d.get('active_lane_fraction'), d['clocks']['sm_mhz'])" | tee -a gpurun_out/${TAG}_ab.log
    done; done; done ;;
ncu)
    CFG=$1; KRE=${2:-track_kernel}; shift 2 || shift $#
    export BENCH_ALLOW_FEW_WARMUP=1
    timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
        --log-file gpurun_out/${TAG}_${CFG}_launches.csv \
        python bench.py --config $CFG --steps 2 --warmup 1 --no-cpu-baseline --no-gather-bench --no-parity \
        --no-lengths "$@" > gpurun_out/${TAG}_${CFG}_launches_bench.log 2>&1
    timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"$KRE" -s 1 -c 1 \
        -o gpurun_out/${TAG}_${CFG}_prof -f \
        python bench.py --config $CFG --steps 1 --warmup 1 --no-cpu-baseline --no-gather-bench --no-parity \
        --no-lengths "$@" > gpurun_out/${TAG}_${CFG}_prof.log 2>&1
    ls -la gpurun_out | tail -5 ;;
*)
    sed -n 2,10p "$0"; exit 2 ;;
esac
