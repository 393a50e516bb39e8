set -x
for mb in 5 6 8; do
PT_LIB=$PWD/scripts/libpt_mb$mb.so timeout 300 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-gather-bench 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('mb$mb', d['value']/1e9, d['roofline']['kernel_ms'])"
done
timeout 300 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-gather-bench 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('mb1', d['value']/1e9, d['roofline']['kernel_ms'])"
timeout 300 python bench.py --config c4 --steps 2 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 > gpurun_out/bench_c4.json; cat gpurun_out/bench_c4.json | cut -c1-2000
