#!/bin/bash
# A/B of tuning knobs then the GPU parity suite: bash tools/gpu_ab.sh TAG SPECS "k=v k=v" "k=v" ...
tag=$1; specs=$2; shift 2
mkdir -p gpurun_out
{
for tk in "$@"; do
  STM_WATCHDOG_S=60 timeout 900 python tools/perf.py $specs reps=3 $tk 2>&1 | grep -v WATCHDOG
done
} > gpurun_out/ab_$tag.log 2>&1
cat gpurun_out/ab_$tag.log
if [ -z "$NO_PYTEST" ]; then
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_$tag.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu_$tag.log
fi
