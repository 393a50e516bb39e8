# A/B of the record layout (PT_BRICK = brick log2 edge, 0 = raster) on c3 and c4, plus the
# parity tests under the bricked layout.
set -x
for b in 3 0 2 4 3; do
  PT_BRICK=$b timeout 600 python bench.py --config c3 --steps 3 --warmup 3 --no-cpu-baseline --no-gather-bench --tag brick$b > gpurun_out/brick_c3_$b.json 2>gpurun_out/brick_c3_$b.err
  python -c "import json;d=json.loads(open('gpurun_out/brick_c3_$b.json').read().strip().splitlines()[-1]);print('c3 brick $b', d['value']/1e9, d['roofline']['frac'])"
done
for b in 0 3; do
  PT_BRICK=$b timeout 600 python bench.py --config c4 --steps 3 --warmup 3 --no-cpu-baseline --no-gather-bench > gpurun_out/brick_c4_$b.json 2>gpurun_out/brick_c4_$b.err
  python -c "import json;d=json.loads(open('gpurun_out/brick_c4_$b.json').read().strip().splitlines()[-1]);print('c4 brick $b', d['value']/1e9)"
done
PT_BRICK=3 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_variants.py tests/test_gpu_ablations.py -x -q > gpurun_out/pytest_brick3.log 2>&1; tail -3 gpurun_out/pytest_brick3.log
