#!/bin/bash
# quick correctness + timing check: bash tools/gpu_check.sh tag [pytest -k expr]
tag=${1:-chk}
mkdir -p gpurun_out
{
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
timeout 1500 python -m pytest tests -m gpu -x -q --durations=12 ${2:+-k "$2"} 2>&1 | tail -20
timeout 600 python tools/perf.py c5:k5,c5:k6_minus_e,c2:k4,c2:c4,c3:k5,c4:c6:vi reps=3
} > gpurun_out/check_$tag.log 2>&1
cat gpurun_out/check_$tag.log
