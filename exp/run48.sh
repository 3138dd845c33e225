export PYTORCH_NO_CUDA_MEMORY_CACHING=1
timeout 2400 compute-sanitizer --tool memcheck --print-limit 20 python exp/sanitize_big.py > gpurun_out/sanitize_big_nocache.log 2>&1; echo big=$?; tail -8 gpurun_out/sanitize_big_nocache.log
timeout 1500 compute-sanitizer --tool memcheck --print-limit 20 python exp/sanitize.py xs > gpurun_out/sanitize_xs_nocache.log 2>&1; echo xs=$?; tail -4 gpurun_out/sanitize_xs_nocache.log
timeout 1500 compute-sanitizer --tool memcheck --print-limit 20 python exp/sanitize.py rs > gpurun_out/sanitize_rs_nocache.log 2>&1; echo rs=$?; tail -4 gpurun_out/sanitize_rs_nocache.log
