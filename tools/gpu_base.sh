#!/bin/bash
# Baseline pass: GPU parity tests, profile-bucket timings of the key workloads, bench.
tag=${1:-b}
mkdir -p gpurun_out
export STM_WATCHDOG_S=${STM_WATCHDOG_S:-60}
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_$tag.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu_$tag.log
STM_LIB_PATH=variants/libstm_prof.so timeout 900 python tools/perf.py c5:k5,c5:k6_minus_e,c2:k4,c2:c4,c3:k5,c3:house reps=2 > gpurun_out/prof_$tag.log 2>&1
grep -v WATCHDOG gpurun_out/prof_$tag.log
timeout 900 python tools/perf.py c5:k5,c5:k6_minus_e,c2:k4,c2:c4,c3:k5,c3:house,c4:c6:vi reps=3 > gpurun_out/perf_$tag.log 2>&1
grep -v WATCHDOG gpurun_out/perf_$tag.log
timeout 900 python bench.py > gpurun_out/bench_$tag.json 2> gpurun_out/bench_$tag.err; echo "bench rc=$?"; cut -c1-400 gpurun_out/bench_$tag.json
