#!/bin/bash
# tuning/variant A/B on chosen queries: bash tools/gpu_ab3.sh tag SPECS "tuning1" "tuning2" ...
# a tuning of the form "lib=PATH ..." loads that variant library (STM_LIB_PATH)
tag=$1; specs=$2; shift 2
mkdir -p gpurun_out
{
for t in "$@"; do
  echo "== $t"
  lib=""; args=""
  for kv in $t; do case $kv in lib=*) lib=${kv#lib=};; *) args="$args $kv";; esac; done
  STM_LIB_PATH=$lib timeout 300 python tools/perf.py $specs reps=3 $args
done
} > gpurun_out/ab_$tag.log 2>&1
cat gpurun_out/ab_$tag.log
