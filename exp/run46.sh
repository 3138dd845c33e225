timeout 1500 compute-sanitizer --tool memcheck --print-limit 20 python exp/sanitize.py xs > gpurun_out/sanitize_xs.log 2>&1; echo xs=$?; tail -25 gpurun_out/sanitize_xs.log
timeout 1500 compute-sanitizer --tool memcheck --print-limit 20 python exp/sanitize.py rs > gpurun_out/sanitize_rs.log 2>&1; echo rs=$?; tail -12 gpurun_out/sanitize_rs.log
