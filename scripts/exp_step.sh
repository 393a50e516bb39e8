set -x
PT_LIB=$PWD/scripts/libpt_cp37.so timeout 900 python -m pytest tests -m gpu -q -x -k "not whole_brain" > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
run() { timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-gather-bench "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('RES', sys.argv[1:], d['value']/1e9, d['ms_per_step'], d['roofline']['kernel_ms'])" "$@"; }
for cp in 1 8 37 148; do PT_LIB=$PWD/scripts/libpt_cp$cp.so run --config c3 --tag cp$cp; done
for cp in 1 37; do PT_LIB=$PWD/scripts/libpt_cp$cp.so run --config c4 --tag cp$cp; done
