timeout 2400 compute-sanitizer --tool memcheck --print-limit 20 python exp/sanitize_big.py > gpurun_out/sanitize_big.log 2>&1; echo big=$?; tail -8 gpurun_out/sanitize_big.log
