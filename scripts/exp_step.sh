set -x
run() { timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-gather-bench "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('RES', sys.argv[1:], d['value']/1e9, d['ms_per_step'], d['roofline']['kernel_ms'])" "$@"; }
for g in 8 16 32 64; do PT_LIB=$PWD/scripts/libpt_g$g.so run --config c3 --tag g$g; done
for g in 8 16 32; do PT_LIB=$PWD/scripts/libpt_g$g.so run --config c4 --tag g$g; done
