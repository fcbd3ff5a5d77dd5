#!/bin/bash
# round-2 check: dist tests, full GPU suite, bench (N=1): bash tools/gpu_round2.sh tag
tag=${1:-r2}
mkdir -p gpurun_out
{
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests/test_gpu_dist.py -x -q 2>&1 | tail -15
timeout 1500 python -m pytest tests -m gpu -x -q ${PYTEST_EXTRA} 2>&1 | tail -15
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench_$tag.json 2> gpurun_out/bench_$tag.err; echo bench rc=$?
tail -30 gpurun_out/bench_$tag.err
} > gpurun_out/round_$tag.log 2>&1
cat gpurun_out/round_$tag.log
