#!/bin/bash
mkdir -p gpurun_out
python -m paper_conf_sc_weij22_b200.build > /dev/null
timeout 900 python tools/census.py c1:5 c1:5:vi c1:6:vi c2:4 c3:4 > gpurun_out/census2.log 2>&1
echo rc=$?; cut -c1-120 gpurun_out/census2.log
timeout 900 python -m pytest tests/test_gpu_parity.py -k "cost_order or motif" -x -q > gpurun_out/pytest_next2.log 2>&1
echo "pytest rc=$?"; tail -2 gpurun_out/pytest_next2.log
