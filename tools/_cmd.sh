mkdir -p gpurun_out
bash tools/gpu_var2.sh d1 c5:k5,c5:k6_minus_e,c3:k5,c2:c4 "cur" "cur|drive_ratio=2" "cur|drive_ratio=4" "cur|drive_ratio=8" "occ64" "occ56|block_warps=14" "occ64|drive_ratio=4"
timeout 900 compute-sanitizer --tool memcheck --print-limit 10 python tools/sanitize.py list > gpurun_out/sanitize_memcheck_list.log 2>&1; echo "memcheck list rc=$?"; grep -E "SANITIZE|ERROR SUMMARY|list" gpurun_out/sanitize_memcheck_list.log | head
