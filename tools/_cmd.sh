bash tools/gpu_var2.sh sd2 c5:k5,c5:k6_minus_e,c3:k5,c2:k4 "cur" "s0d0" "cur" "s0d0"
timeout 900 compute-sanitizer --tool racecheck --print-limit 10 python tools/sanitize.py nosteal > gpurun_out/sanitize_racecheck_nosteal_v3.log 2>&1; echo "racecheck rc=$?"; grep -E "SANITIZE|SUMMARY|Warning|Error" gpurun_out/sanitize_racecheck_nosteal_v3.log | head -12
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_sd2.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu_sd2.log
