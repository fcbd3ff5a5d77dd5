#!/bin/bash
# round-2 re-entry check: full GPU suite + bench + ncu evidence: bash tools/gpu_r2c.sh tag
tag=${1:-r2c}
bash tools/gpu_round2.sh $tag
bash tools/gpu_final_prof.sh $tag
