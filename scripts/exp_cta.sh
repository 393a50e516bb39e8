set -x
PT_LIB=$PWD/scripts/libpt_cta1024.so timeout 900 python -m pytest tests -m gpu -q -x -k "not whole_brain" > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
run() { timeout 300 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-gather-bench "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('RES', sys.argv[1:], d['value']/1e9, d['roofline']['kernel_ms'], d['active_lane_fraction'])" "$@"; }
for c in 1024 512 256; do
PT_LIB=$PWD/scripts/libpt_cta$c.so run --config c3 --tag cta$c
PT_LIB=$PWD/scripts/libpt_cta$c.so run --config c4 --tag cta$c
done
PT_LIB=$PWD/scripts/libpt_cta1024.so run --config c3 --no-map --tag cta1024
