#!/bin/bash
# final evidence: ncu --set full of the C5 launches + the bench launch list: bash tools/gpu_final_prof.sh tag
tag=${1:-f}
mkdir -p gpurun_out
{
for q in k6_minus_e k5; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:stm_count_kernel -s 1 -c 1 \
     -f -o gpurun_out/ncu_${tag}_$q python tools/prof_run.py c5 $q > gpurun_out/ncu_${tag}_$q.log 2>&1
  echo "ncu $q rc=$?"
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${tag}.csv \
   python bench.py --steps 2 --warmup 3 --no-per-config --no-cpu-baseline --no-e2e > gpurun_out/launches_${tag}.log 2>&1
echo "launches rc=$?"
} > gpurun_out/final_prof_$tag.log 2>&1
cat gpurun_out/final_prof_$tag.log
