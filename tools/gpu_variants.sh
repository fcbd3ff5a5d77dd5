#!/bin/bash
# usage (under gpurun): bash tools/gpu_variants.sh TAG SPECS v0 v1 ...   (SPECS = tools/perf.py spec list)
tag=$1; specs=$2; shift 2
mkdir -p gpurun_out
export STM_WATCHDOG_S=${STM_WATCHDOG_S:-30}
for v in "$@"; do
  echo "== variant $v"
  STM_LIB_PATH=variants/libstm_$v.so timeout 600 python tools/perf.py $specs reps=3
done > gpurun_out/variants_$tag.log 2>&1
cat gpurun_out/variants_$tag.log
