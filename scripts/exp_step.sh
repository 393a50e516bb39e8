set -x
timeout 900 python -m pytest tests -m gpu -q -x -k "paper" > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
run() { timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-gather-bench "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('RES', sys.argv[1:], d['value']/1e9, d['ms_per_step'], d['roofline']['kernel_ms'], d.get('lengths'))" "$@"; }
run --config c3 --tag base
for pf in 128 256; do PT_LIB=$PWD/scripts/libpt_l2p$pf.so run --config c3 --tag l2p$pf; done
for pf in 256; do PT_LIB=$PWD/scripts/libpt_l2p$pf.so run --config c4 --tag l2p$pf; done
run --config c4 --tag base
run --config d1 --tag paper
run --config d2 --tag paper
