timeout 900 compute-sanitizer --tool racecheck --print-limit 10 python tools/sanitize.py nosteal > gpurun_out/sanitize_racecheck_nosteal_v4.log 2>&1; echo "racecheck rc=$?"; grep -E "SANITIZE|SUMMARY|Warning|Error" gpurun_out/sanitize_racecheck_nosteal_v4.log | head -6
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_f2.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu_f2.log
bash tools/gpu_bench.sh f2
bash tools/gpu_ncu.sh f2 c5 k6_minus_e
