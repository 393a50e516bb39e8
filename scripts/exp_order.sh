set -x
timeout 900 python -m pytest tests -m gpu -q -x -k "not whole_brain" > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
for fl in 0 512; do
for cfg in c3 c4; do
timeout 300 python bench.py --config $cfg --steps 2 --warmup 3 --no-cpu-baseline --no-gather-bench --track-flags $fl 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('flags$fl', '$cfg', d['value']/1e9, d['roofline']['kernel_ms'], d['e2e']['value']/1e9)"
done; done
