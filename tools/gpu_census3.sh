#!/bin/bash
mkdir -p gpurun_out
python -m paper_conf_sc_weij22_b200.build > /dev/null
timeout 900 python -m pytest tests/test_gpu_parity.py -k "cost_order or motif" -x -q > gpurun_out/pytest_next3.log 2>&1
echo "pytest rc=$?"; tail -2 gpurun_out/pytest_next3.log
timeout 900 python tools/census.py c1:5 c1:5:vi c1:6:vi c2:4 > gpurun_out/census3.log 2>&1
echo rc=$?; grep -v WATCHDOG gpurun_out/census3.log | cut -c1-100
S=c2:c4:cost,c2:tailed_triangle,c2:tailed_triangle:cost,c4:c6:vi:cost,c4:prism:cost,c5:c4:cost,c3:c5:cost
STM_WATCHDOG_S=60 timeout 900 python tools/perf.py $S reps=3 2>&1 | grep -v WATCHDOG > gpurun_out/ab_cost_order_v3.log
grep best gpurun_out/ab_cost_order_v3.log
