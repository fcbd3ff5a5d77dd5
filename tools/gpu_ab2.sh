#!/bin/bash
# tuning A/B on the main queries: bash tools/gpu_ab2.sh tag "tuning1" "tuning2" ...
tag=$1; shift
mkdir -p gpurun_out
{
for t in "$@"; do
  echo "== $t"
  timeout 300 python tools/perf.py c5:k5,c5:k6_minus_e,c3:k5,c2:k4,c2:c4,c4:c6:vi reps=3 $t
done
} > gpurun_out/ab_$tag.log 2>&1
cat gpurun_out/ab_$tag.log
