# r01j: 6-step refill rounds as default (PT_ROUND_BLOCKS=2): full GPU suite, smoke, refill-threshold A/B, default bench line
set -x
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r01j_pytest_gpu_final.log 2>&1; tail -3 gpurun_out/r01j_pytest_gpu_final.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r01j_smoke_final.log 2>&1; tail -2 gpurun_out/r01j_smoke_final.log
for rep in 1 2; do
for lib in default rb1 rb2m1 rb2m4; do
for cfg in c3 c4; do
if [ $lib = default ]; then L=$PWD/paper_conf_ipps_xuzwrwxgxy12_b200/libpt.so; else L=$PWD/scripts/libpt_$lib.so; fi
PT_LIB=$L timeout 300 python bench.py --config $cfg --steps 3 --warmup 3 --no-cpu-baseline --no-gather-bench 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$lib', '$cfg', d['value']/1e9, d['roofline']['kernel_ms'], d['active_lane_fraction'], d['clocks']['sm_mhz'])"
done; done; done
timeout 900 python bench.py > gpurun_out/r01j_bench_c3_final.json 2> gpurun_out/r01j_bench_c3_final.err; cut -c1-400 gpurun_out/r01j_bench_c3_final.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r01j_c3_launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/r01j_ncu_bench.log 2>&1; tail -2 gpurun_out/r01j_ncu_bench.log
