set -x
PT_LIB=$PWD/scripts/libpt_mb5.so timeout 900 python -m pytest tests -m gpu -q -x -k "not whole_brain" > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
for mb in 1 5 6; do
for cfg in c3 c4; do
PT_LIB=$PWD/scripts/libpt_mb$mb.so timeout 300 python bench.py --config $cfg --steps 2 --warmup 3 --no-cpu-baseline --no-gather-bench 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('mb$mb', '$cfg', d['value']/1e9, d['roofline']['kernel_ms'], d['active_lane_fraction'])"
done; done
