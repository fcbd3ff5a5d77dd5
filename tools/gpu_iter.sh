#!/bin/bash
# iteration check: focused parity subset + A/B + scaling probe: bash tools/gpu_iter.sh tag "pytest -k expr" "tuning1" ...
tag=$1; kexpr=$2; shift 2
mkdir -p gpurun_out
{
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
timeout 900 python -m pytest tests -m gpu -x -q -k "$kexpr" 2>&1 | tail -6
for t in "$@"; do
  echo "== $t"
  timeout 300 python tools/perf.py c5:k5,c5:k6_minus_e,c3:k5,c2:k4,c2:c4,c4:c6:vi reps=3 $t
done
} > gpurun_out/iter_$tag.log 2>&1
cat gpurun_out/iter_$tag.log
