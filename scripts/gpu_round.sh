set -x
timeout 1500 python -m pytest tests -m gpu -q -k "not whole_brain" > gpurun_out/pytest_gpu.log 2>&1; tail -15 gpurun_out/pytest_gpu.log
CFG=c3 TAG=r01 timeout 1200 bash scripts/profile.sh
