# PT_KERNEL_SPEC ablation parity + hit statistics; c5 (HCP-scale) bench line with emulated 2/4/8-rank scaling
set -x
timeout 900 python -m pytest tests/test_gpu_spec.py -x -q > gpurun_out/spec2_pytest.log 2>&1; tail -5 gpurun_out/spec2_pytest.log
timeout 600 python bench.py --config c3 --steps 3 --warmup 3 --no-cpu-baseline --no-gather-bench --track-flags 131072 > gpurun_out/spec2_c3.json 2>gpurun_out/spec2_c3.err; python -c "import json;d=json.loads(open('gpurun_out/spec2_c3.json').read().strip().splitlines()[-1]);print('spec',d['value']/1e9,d['spec_step_fraction'],d['steps_per_lane_iteration'])"
timeout 1800 python bench.py --config c5 --emulate-ranks 2,4,8 > gpurun_out/c5_bench.json 2>gpurun_out/c5_bench.err; cut -c1-1500 gpurun_out/c5_bench.json; tail -3 gpurun_out/c5_bench.err
