# r01j re-entry check: full GPU suite, smoke, default bench line (c3), ncu launch list
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r01j_pytest_gpu.log 2>&1; tail -5 gpurun_out/r01j_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r01j_smoke.log 2>&1; tail -2 gpurun_out/r01j_smoke.log
timeout 900 python bench.py > gpurun_out/r01j_bench_c3.json 2> gpurun_out/r01j_bench_c3.err; cut -c1-600 gpurun_out/r01j_bench_c3.json
