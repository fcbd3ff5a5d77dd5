#!/bin/bash
# usage (under gpurun): bash tools/gpu_tune.sh TAG SPECS "k=v k=v" "k=v" ...   (tuning sweeps on the in-tree lib)
tag=$1; specs=$2; shift 2
mkdir -p gpurun_out
export STM_WATCHDOG_S=${STM_WATCHDOG_S:-30}
for t in "$@"; do
  echo "== tuning $t"
  timeout 600 python tools/perf.py $specs $t reps=3
done > gpurun_out/tune_$tag.log 2>&1
cat gpurun_out/tune_$tag.log
