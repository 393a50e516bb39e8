# Record-layout follow-up: brick edge 16/32, and the occupancy / claim sweeps redone under
# the bricked layout (experiment builds under scripts/).
run() { timeout 400 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-gather-bench "$@" 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('RES', sys.argv[1:], round(d['value']/1e9,2), round(d['roofline']['frac'],4), d['roofline']['kernel_ms'], d['active_lane_fraction'])" "$@"; }
PT_BRICK=4 run --config c3 --tag b4
PT_BRICK=5 run --config c3 --tag b5
PT_BRICK=4 PT_LIB=$PWD/scripts/libpt_slots2.so run --config c3 --tag b4_slots2
PT_BRICK=4 PT_LIB=$PWD/scripts/libpt_spc1.so run --config c3 --tag b4_spc1
PT_BRICK=4 PT_LIB=$PWD/scripts/libpt_spc8.so run --config c3 --tag b4_spc8
PT_BRICK=4 run --config c3 --tag b4_again
PT_BRICK=4 run --config c3 --no-map --tag b4_nomap
PT_BRICK=4 run --config c4 --tag b4_c4
PT_BRICK=4 run --config c3 --track-flags 256 --tag b4_simple
