#!/bin/bash
# variant A/B: bash tools/gpu_var2.sh TAG SPECS "variant|k=v k=v" ...
tag=$1; specs=$2; shift 2
mkdir -p gpurun_out
for vt in "$@"; do
  v=${vt%%|*}; tk=${vt#*|}; [ "$tk" = "$vt" ] && tk=""
  echo "== variant $v $tk"
  STM_WATCHDOG_S=60 STM_LIB_PATH=variants/libstm_$v.so timeout 600 python tools/perf.py $specs reps=3 $tk 2>&1 | grep -v WATCHDOG
done > gpurun_out/var_$tag.log 2>&1
cat gpurun_out/var_$tag.log
