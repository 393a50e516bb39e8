set -x
run() { timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-gather-bench "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('RES', sys.argv[1:], d['value']/1e9, d['ms_per_step'], d['roofline']['kernel_ms'])" "$@"; }
for v in h0p0 h1p0 h0p1; do PT_LIB=$PWD/scripts/libpt_$v.so run --config c3 --tag $v; done
for v in h0p0 h1p0; do PT_LIB=$PWD/scripts/libpt_$v.so run --config c4 --tag $v; done
