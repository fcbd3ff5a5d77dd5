#!/bin/bash
# Build A/B variant libraries into variants/ (git-ignored .so; they travel with gpurun).
# usage: bash tools/build_variants.sh "name:DEF=1,DEF2=0" ...
mkdir -p variants
for spec in "$@"; do
  name=${spec%%:*}; defs=${spec#*:}
  python paper_conf_sc_weij22_b200/build.py --force --out=variants/libstm_$name.so ${defs//,/ } > variants/build_$name.log 2>&1 &
done
wait
for spec in "$@"; do name=${spec%%:*}; echo "$name: $(grep -A2 'stm_count_kernel' variants/build_$name.log | grep -E 'stack|registers' | tr '\n' ' ')"; done
