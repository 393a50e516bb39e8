# occupancy re-sweep under bricks: 1 x 1024 threads per SM (default, 62 regs) vs 2 x 640 (48 regs) vs 2 x 768 (40 regs)
set -x
PT_LIB=$PWD/scripts/libpt_t640x2.so timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "c1_full or c2_dispersed or paths_bit" > gpurun_out/exp_threads_pytest.log 2>&1; tail -2 gpurun_out/exp_threads_pytest.log
for rep in 1 2; do
for lib in paper_conf_ipps_xuzwrwxgxy12_b200/libpt.so scripts/libpt_t640x2.so scripts/libpt_t768x2.so; do
for cfg in c3 c4; do
PT_LIB=$PWD/$lib timeout 300 python bench.py --config $cfg --steps 2 --warmup 3 --no-cpu-baseline --no-gather-bench 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('RES', '$lib', '$cfg', round(d['value']/1e9,2), round(d['roofline']['kernel_ms'],1), d['active_lane_fraction'])"
done; done; done
