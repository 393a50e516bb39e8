# speculative-gather kernel: parity (full GPU suite exercises it as the default kernel), A/B bench vs ROUND3
set -x
timeout 1500 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/spec_pytest_parity.log 2>&1; tail -5 gpurun_out/spec_pytest_parity.log
for i in 1 2; do
timeout 600 python bench.py --config c3 --steps 3 --warmup 3 --no-cpu-baseline --no-gather-bench > gpurun_out/spec_c3_$i.json 2>gpurun_out/spec_c3_$i.err; python -c "import json;d=json.loads(open('gpurun_out/spec_c3_$i.json').read().strip().splitlines()[-1]);print('spec',d['value']/1e9,d['active_lane_fraction'],d['roofline']['frac'])"
timeout 600 python bench.py --config c3 --steps 3 --warmup 3 --no-cpu-baseline --no-gather-bench --track-flags 131072 > gpurun_out/r3_c3_$i.json 2>gpurun_out/r3_c3_$i.err; python -c "import json;d=json.loads(open('gpurun_out/r3_c3_$i.json').read().strip().splitlines()[-1]);print('round3',d['value']/1e9,d['active_lane_fraction'])"
done
timeout 600 python bench.py --config c4 --steps 3 --warmup 3 --no-cpu-baseline --no-gather-bench > gpurun_out/spec_c4.json 2>gpurun_out/spec_c4.err; python -c "import json;d=json.loads(open('gpurun_out/spec_c4.json').read().strip().splitlines()[-1]);print('spec c4',d['value']/1e9)"
