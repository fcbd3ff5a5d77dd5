#!/bin/bash
# NEXT-2 on the GPU: cost-order parity tests, then greedy vs cost-order timing A/B.
mkdir -p gpurun_out
python -m paper_conf_sc_weij22_b200.build > /dev/null
timeout 900 python -m pytest tests/test_gpu_parity.py -k cost_order -x -q > gpurun_out/pytest_cost_order.log 2>&1
echo "pytest rc=$?"; tail -3 gpurun_out/pytest_cost_order.log
S=c2:c4,c2:c4:cost,c2:c4:vi,c2:c4:vi:cost,c4:c6:vi,c4:c6:vi:cost,c4:w6,c4:w6:cost,c4:prism,c4:prism:cost,c3:house,c3:house:cost,c3:c5,c3:c5:cost,c4:c7:vi,c4:c7:vi:cost,c5:c4,c5:c4:cost
STM_WATCHDOG_S=60 timeout 1500 python tools/perf.py $S reps=3 > gpurun_out/ab_cost_order.log 2>&1
cat gpurun_out/ab_cost_order.log
