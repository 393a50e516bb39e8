# r01i final evidence: c3 / c4 bench lines with emulated 2/4/8-rank scaling, ncu launch list + full capture of the tracking kernel (c3)
set -x
timeout 1200 python bench.py --config c3 --emulate-ranks 2,4,8 > gpurun_out/r01i_bench_c3_emulated.json 2> gpurun_out/r01i_bench_c3_emulated.err; cut -c1-400 gpurun_out/r01i_bench_c3_emulated.json
timeout 1200 python bench.py --config c4 --emulate-ranks 2,4,8 > gpurun_out/r01i_bench_c4_emulated.json 2> gpurun_out/r01i_bench_c4_emulated.err; cut -c1-400 gpurun_out/r01i_bench_c4_emulated.json
CFG=c3 TAG=r01i timeout 1500 bash scripts/profile.sh > gpurun_out/r01i_profile.log 2>&1; tail -5 gpurun_out/r01i_profile.log
