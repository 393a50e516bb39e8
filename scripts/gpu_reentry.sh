# re-entry check: full GPU suite, smoke, default bench line (c3)
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_r01i.log 2>&1; tail -5 gpurun_out/pytest_gpu_r01i.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r01i.log 2>&1; tail -2 gpurun_out/smoke_r01i.log
timeout 900 python bench.py > gpurun_out/bench_c3_r01i.json 2> gpurun_out/bench_c3_r01i.err; cut -c1-600 gpurun_out/bench_c3_r01i.json
