run() { timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-gather-bench "$@" 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); e=d.get('emulated_scaling') or {}
print('RES', sys.argv[1:], round(d['value']/1e9,2), {k: (round(v['projected_value']/1e9,1), round(max(v['shard_ms']),1), round(v['imbalance_max_over_mean'],4)) for k,v in e.items()})" "$@"; }
PT_SHARD_BLOCK=512 run --config c3 --emulate-ranks 4,8 --tag block512
PT_SHARD_BLOCK=2048 run --config c3 --emulate-ranks 8 --tag block2048
PT_SHARD_BLOCK=1024 run --config c3 --emulate-ranks 8 --tag block1024_again
