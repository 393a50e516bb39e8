# experiment: brick record index as a sum of per-axis affine terms (PT_REC_AFFINE=1, scripts/libpt_aff.so) vs default; parity + A/B x2 same box
set -x
PT_LIB=$PWD/scripts/libpt_aff.so timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x > gpurun_out/r01j_pytest_gpu_aff.log 2>&1; tail -2 gpurun_out/r01j_pytest_gpu_aff.log
for rep in 1 2 3; do
for lib in default aff; do
for cfg in c3 c4; do
if [ $lib = default ]; then L=$PWD/paper_conf_ipps_xuzwrwxgxy12_b200/libpt.so; else L=$PWD/scripts/libpt_$lib.so; fi
PT_LIB=$L timeout 300 python bench.py --config $cfg --steps 3 --warmup 3 --no-cpu-baseline --no-gather-bench 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$lib', '$cfg', d['value']/1e9, d['roofline']['kernel_ms'], d['active_lane_fraction'], d['clocks']['sm_mhz'])"
done; done; done
