#!/bin/bash
# final state: full GPU suite, smoke, bench (one call)
mkdir -p gpurun_out
python -m paper_conf_sc_weij22_b200.build > /dev/null
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_final2.log 2>&1
echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu_final2.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_final2.log 2>&1; echo "smoke rc=$?"
timeout 900 python bench.py > gpurun_out/bench_final2.json 2> gpurun_out/bench_final2.err; echo "bench rc=$?"; cut -c1-1500 gpurun_out/bench_final2.json
