#!/bin/bash
# Full GPU parity suite (after a rebuild) -> gpurun_out/pytest_gpu_$1.log
mkdir -p gpurun_out
python -m paper_conf_sc_weij22_b200.build > /dev/null
timeout 2400 python -m pytest tests -m gpu -q --durations=15 > gpurun_out/pytest_gpu_$1.log 2>&1
echo "pytest rc=$?"; tail -25 gpurun_out/pytest_gpu_$1.log
