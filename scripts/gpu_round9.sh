set -x
timeout 900 python bench.py --config m2 --steps 5 --warmup 3 > gpurun_out/bench_m2.json 2> gpurun_out/bench_m2.err; cat gpurun_out/bench_m2.json
timeout 600 python bench.py --config m2 --impl reference --steps 2 --warmup 1 > gpurun_out/bench_m2_ref.json 2>&1; tail -1 gpurun_out/bench_m2_ref.json
PT_LIB=$PWD/scripts/libpt_norunlen.so timeout 600 python scripts/ablations.py --config c3 --reps 1 --only main > gpurun_out/ablation_norunlen.log 2>&1; tail -3 gpurun_out/ablation_norunlen.log
timeout 600 python scripts/ablations.py --config c3 --reps 1 --only main > gpurun_out/ablation_runlen.log 2>&1; tail -3 gpurun_out/ablation_runlen.log
timeout 600 python bench.py --config c3 --steps 2 --warmup 3 --no-map --no-cpu-baseline --no-gather-bench > gpurun_out/bench_c3_nomap.json 2>&1; tail -1 gpurun_out/bench_c3_nomap.json | cut -c1-300
