STM_LIB_PATH=variants/libstm_prof.so python tools/perf.py c5:k5,c5:k6_minus_e,c2:k4,c2:c4,c3:k5 reps=2 > gpurun_out/prof_a5.log 2>&1
grep -v WATCHDOG gpurun_out/prof_a5.log
