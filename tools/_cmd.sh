mkdir -p gpurun_out
run() { tool=$1; mode=$2; tag=$3; echo "== $tool $mode $tag"; timeout 900 compute-sanitizer --tool $tool --print-limit 10 python tools/sanitize.py $mode > gpurun_out/sanitize_${tool}_${mode}$tag.log 2>&1; echo "rc=$?"; grep -E "SANITIZE|ERROR SUMMARY|RACECHECK SUMMARY|Error:|list|occupancy" gpurun_out/sanitize_${tool}_${mode}$tag.log | head -8; }
CUDA_MODULE_LOADING=EAGER run memcheck list _eager
run racecheck nosteal _v2
run racecheck count _v2
python tools/sanitize.py list
