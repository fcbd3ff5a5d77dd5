STM_WATCHDOG_S=60 timeout 900 python tools/perf.py c5:k5,c5:k6_minus_e,c3:k5,c2:k4,c2:c4 reps=3 2>&1 | grep -v WATCHDOG
for b in 64 256 1024; do STM_WATCHDOG_S=60 timeout 900 python tools/perf.py c5:k5,c5:k6_minus_e reps=3 bitmap_budget_mb=$b 2>&1 | grep -v WATCHDOG; done
timeout 1500 python -m pytest tests -m gpu -x -q --durations=30 > gpurun_out/pytest_gpu_s1.log 2>&1; echo "pytest rc=$?"; tail -45 gpurun_out/pytest_gpu_s1.log
