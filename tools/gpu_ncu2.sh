#!/bin/bash
# phase profile + ncu --set full of the C5 launches: bash tools/gpu_ncu2.sh tag
tag=${1:-n}
mkdir -p gpurun_out
{
STM_LIB_PATH=variants/libstm_prof.so timeout 300 python tools/perf.py c5:k5,c5:k6_minus_e reps=2
for q in k6_minus_e k5; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:stm_count_kernel -s 1 -c 1 \
     -f -o gpurun_out/ncu_${tag}_$q python tools/prof_run.py c5 $q > gpurun_out/ncu_${tag}_$q.log 2>&1
  echo "ncu $q rc=$?"
done
} > gpurun_out/ncu_$tag.log 2>&1
cat gpurun_out/ncu_$tag.log
