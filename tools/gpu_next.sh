#!/bin/bash
# NEXT-2 hysteresis + NEXT-3 census on the GPU: parity subset, A/B rows, census timing.
mkdir -p gpurun_out
python -m paper_conf_sc_weij22_b200.build > /dev/null
timeout 1200 python -m pytest tests/test_gpu_parity.py -k "cost_order or motif" -x -q > gpurun_out/pytest_next.log 2>&1
echo "pytest rc=$?"; tail -3 gpurun_out/pytest_next.log
S=c4:c6:vi,c4:c6:vi:cost,c4:c7:vi:cost,c4:prism:cost,c2:c4:cost,c5:c4:cost,c3:c5:cost
STM_WATCHDOG_S=60 timeout 900 python tools/perf.py $S reps=3 2>&1 | grep -v WATCHDOG > gpurun_out/ab_cost_order_v2.log
cat gpurun_out/ab_cost_order_v2.log
timeout 900 python tools/census.py c1:5 c1:6:vi c2:4 c2:4:vi > gpurun_out/census.log 2>&1
cat gpurun_out/census.log | cut -c1-200
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -3 gpurun_out/smoke.log
