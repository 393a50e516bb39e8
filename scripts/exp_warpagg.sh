# ablation (iv) warp-aggregated counting (PT_RUNLEN=2, scripts/libpt_rl2.so) vs default run-length RED (A/B, same box)
set -x
PT_LIB=$PWD/scripts/libpt_rl2.so timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x > gpurun_out/r01j_pytest_gpu_rl2.log 2>&1; tail -3 gpurun_out/r01j_pytest_gpu_rl2.log
for rep in 1 2; do
for lib in default rl2; do
for cfg in c3 c4; do
if [ $lib = default ]; then L=$PWD/paper_conf_ipps_xuzwrwxgxy12_b200/libpt.so; else L=$PWD/scripts/libpt_$lib.so; fi
PT_LIB=$L timeout 300 python bench.py --config $cfg --steps 3 --warmup 3 --no-cpu-baseline --no-gather-bench 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$lib', '$cfg', d['value']/1e9, d['roofline']['kernel_ms'], d['clocks']['sm_mhz'])"
done; done; done
for lib in default rl2; do
if [ $lib = default ]; then L=$PWD/paper_conf_ipps_xuzwrwxgxy12_b200/libpt.so; else L=$PWD/scripts/libpt_$lib.so; fi
PT_LIB=$L timeout 600 ncu --metrics lts__t_sectors_srcunit_tex_op_red.sum,smsp__inst_executed.sum,gpu__time_duration.sum,smsp__issue_active.avg.pct_of_peak_sustained_active -k regex:track_kernel -c 1 --csv python bench.py --config c3 --steps 1 --warmup 0 --no-cpu-baseline --no-gather-bench --no-per-step-stats > gpurun_out/r01j_ncu_$lib.csv 2>&1; grep -E "red.sum|inst_executed.sum|duration|issue_active" gpurun_out/r01j_ncu_$lib.csv | cut -c1-300
done
