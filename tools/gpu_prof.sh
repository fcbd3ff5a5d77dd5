#!/bin/bash
# per-phase profile (STM_PROFILE build) + plain timings: bash tools/gpu_prof.sh tag
tag=${1:-p}
mkdir -p gpurun_out
{
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 600 python tools/perf.py c5:k5,c5:k6_minus_e reps=3
STM_LIB_PATH=variants/libstm_prof.so timeout 600 python tools/perf.py c5:k5,c5:k6_minus_e reps=2
} > gpurun_out/prof_$tag.log 2>&1
cat gpurun_out/prof_$tag.log
