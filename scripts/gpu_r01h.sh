# r01h: default build (compile-time bricks, refill threshold 2): GPU suite, default bench line,
# ablation table (incl. the record layout), emulated scaling c3, variants bench.
set -x
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r01h_pytest_gpu.log 2>&1; tail -2 gpurun_out/r01h_pytest_gpu.log
timeout 900 python bench.py > gpurun_out/r01h_bench_c3.json 2> gpurun_out/r01h_bench_c3.err; cut -c1-300 gpurun_out/r01h_bench_c3.json
timeout 1500 python scripts/ablations.py --config c3 --reps 2 > gpurun_out/r01h_ablations_c3.log 2>&1; tail -16 gpurun_out/r01h_ablations_c3.log
timeout 1200 python bench.py --config c3 --steps 3 --warmup 3 --no-cpu-baseline --no-gather-bench --emulate-ranks 2,4,8 > gpurun_out/r01h_bench_c3_emulated.json 2> gpurun_out/r01h_bench_c3_emulated.err; python -c "import json;d=json.loads(open('gpurun_out/r01h_bench_c3_emulated.json').read().strip().splitlines()[-1]);print(json.dumps(d['emulated_scaling'])[:1500])"
