#!/bin/bash
# ncu --set full capture of one query launch (the 2nd; the 1st warms up / builds bitmaps)
# usage (under gpurun): bash tools/gpu_ncu.sh TAG CFG PATTERN
tag=$1; cfg=$2; pat=$3
mkdir -p gpurun_out
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:stm_count -s 1 -c 1 -f \
   -o gpurun_out/prof_${cfg}_${pat}_$tag python tools/prof_run.py $cfg $pat > gpurun_out/ncu_$tag.log 2>&1; echo "ncu rc=$?"
tail -3 gpurun_out/ncu_$tag.log
