# NEXT-3 variant kernel: parity suite + throughput of each variant on c3.
set -x
timeout 1500 python -m pytest tests/test_gpu_variants.py -q -x > gpurun_out/pytest_gpu_variants.log 2>&1; tail -15 gpurun_out/pytest_gpu_variants.log
for fl in 32768 2048 4096 6144 14336; do
  timeout 300 python bench.py --config c3 --steps 3 --warmup 3 --no-cpu-baseline --no-gather-bench --track-flags $fl > gpurun_out/bench_var_$fl.json 2> gpurun_out/bench_var_$fl.err
  python -c "import json;d=json.load(open('gpurun_out/bench_var_$fl.json'));print($fl, d['value']/1e9, d['roofline']['kernel_ms'], d.get('active_lane_fraction'))"
done
