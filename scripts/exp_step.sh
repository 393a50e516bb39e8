set -x
PT_LIB=$PWD/scripts/libpt_sl2.so timeout 900 python -m pytest tests -m gpu -q -x -k "not whole_brain" > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
run() { timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-gather-bench "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('RES', sys.argv[1:], d['value']/1e9, d['ms_per_step'], d['roofline']['kernel_ms'], d['active_lane_fraction'])" "$@"; }
for v in sl1 sl2 sl2t640 sl2t704; do PT_LIB=$PWD/scripts/libpt_$v.so run --config c3 --tag $v; done
for v in sl1 sl2; do PT_LIB=$PWD/scripts/libpt_$v.so run --config c4 --tag $v; done
