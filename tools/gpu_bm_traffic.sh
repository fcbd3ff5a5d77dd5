#!/bin/bash
mkdir -p gpurun_out
{
for t in "" "bitmap_budget_mb=96" "bitmap_budget_mb=256" "bitmap_budget_mb=512" "bitmap_min_degree=-1"; do
  echo "== $t"
  timeout 300 python tools/perf.py c5:k6_minus_e,c5:k5 reps=3 $t
  timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum -k regex:stm_count_kernel --csv python tools/perf.py c5:k6_minus_e reps=1 $t 2>/dev/null | grep -E "dram__bytes|gpu__time" | tail -3
done
} > gpurun_out/bm_traffic.log 2>&1
