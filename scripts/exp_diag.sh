set -x
run() { timeout 300 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-gather-bench "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('RES', sys.argv[1:], d['value']/1e9, d['roofline']['kernel_ms'], d['config']['mean_steps_per_streamline'])" "$@"; }
run --config c3 --no-map
run --config c3
run --config c2_dispersed
run --config c2
run --config c4 --no-map
