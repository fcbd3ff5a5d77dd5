#!/bin/bash
# quick A/B timings under gpurun: bash tools/gpu_perf.sh tag
tag=${1:-p}
mkdir -p gpurun_out
export STM_WATCHDOG_S=${STM_WATCHDOG_S:-40}
{
timeout 300 python tools/perf.py c2:k4,c2:c4,c2:c4:vi vertex_order=1
timeout 300 python tools/perf.py c2:k4,c2:c4,c2:c4:vi vertex_order=0
timeout 600 python tools/perf.py c3:k5,c3:house,c3:c5 vertex_order=1
timeout 600 python tools/perf.py c3:k5,c3:house,c3:c5 vertex_order=0
timeout 900 python tools/perf.py c5:k5,c5:k6,c5:k6_minus_e,c5:octahedron,c5:w5,c5:prism,c5:c4 vertex_order=0 reps=2
timeout 300 python tools/perf.py c5:k5 vertex_order=1 reps=2
timeout 600 python tools/perf.py c4:k6_minus_e,c4:w5,c4:c6:vi,c4:w6,c4:c7:vi vertex_order=0
} > gpurun_out/perf_$tag.log 2>&1
cat gpurun_out/perf_$tag.log
