set -x
timeout 1500 python -m pytest tests -m gpu -q -x -k "connectivity or paper or c2_full or paths" > gpurun_out/pytest_gpu.log 2>&1; tail -15 gpurun_out/pytest_gpu.log
run() { timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-gather-bench "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('RES', sys.argv[1:], d['value']/1e9, d['ms_per_step'], d['roofline']['kernel_ms'])" "$@"; }
run --config c3
