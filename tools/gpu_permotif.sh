#!/bin/bash
mkdir -p gpurun_out
python -m paper_conf_sc_weij22_b200.build > /dev/null
timeout 1200 python tools/census_permotif.py c1:6:vi c1:5:vi c1:5 c3:4 c2:4 > gpurun_out/permotif.log 2>&1
echo rc=$?; cat gpurun_out/permotif.log | grep -v WATCHDOG | tail -100
