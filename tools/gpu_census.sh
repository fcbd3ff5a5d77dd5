#!/bin/bash
# census parity + timing: bash tools/gpu_census.sh tag
tag=${1:-c}
mkdir -p gpurun_out
{
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "census" 2>&1 | tail -5
timeout 900 python tools/census.py c1:4 c1:5 c1:5:vi c1:6 c1:6:vi c2:4 c2:4:vi 2>&1
} > gpurun_out/census_$tag.log 2>&1
cat gpurun_out/census_$tag.log
