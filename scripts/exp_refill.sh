# compile-time brick layout + lazy sfix (default build) and the refill-threshold sweep
run() { timeout 400 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-gather-bench "$@" 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('RES', sys.argv[1:], round(d['value']/1e9,2), round(d['roofline']['frac'],4), d['roofline']['kernel_ms'], d['active_lane_fraction'])" "$@"; }
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/pytest_parity_refill.log 2>&1; tail -2 gpurun_out/pytest_parity_refill.log
run --config c3 --tag default
PT_LIB=$PWD/scripts/libpt_rm2.so run --config c3 --tag rm2
PT_LIB=$PWD/scripts/libpt_rm4.so run --config c3 --tag rm4
PT_LIB=$PWD/scripts/libpt_rm8.so run --config c3 --tag rm8
run --config c3 --tag default_again
PT_LIB=$PWD/scripts/libpt_rm4.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "c2 or paths or layout" > gpurun_out/pytest_parity_rm4.log 2>&1; tail -2 gpurun_out/pytest_parity_rm4.log
