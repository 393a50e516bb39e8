# guided tail claims + variant kernel brick index: parity, c3 bench, emulated 8-way shards, variants
run() { timeout 400 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-gather-bench "$@" 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('RES', sys.argv[1:], round(d['value']/1e9,2), round(d['roofline']['frac'],4), d['roofline']['kernel_ms'], d['active_lane_fraction'], json.dumps(d.get('emulated_scaling'))[:900])" "$@"; }
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_variants.py -x -q > gpurun_out/pytest_tail.log 2>&1; tail -2 gpurun_out/pytest_tail.log
run --config c3 --tag tail
run --config c3 --emulate-ranks 8 --tag tail_em8
timeout 900 python scripts/ablations.py --config c3 --reps 1 --only "variant kernel" 2>&1 | tail -3
