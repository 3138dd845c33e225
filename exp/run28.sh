timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_f32.py tests/test_gpu_history.py -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -15 gpurun_out/pytest_gpu.log
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none -k regex:"k_part|k_gather" -c 8 --csv python tools/profile_one.py --config large --sort --reps 1 2>/dev/null | grep -v "^==" | awk -F'","' '{print $5, $13, $15}' | cut -c1-200
timeout 600 python exp/qt2.py large small large-hash 2>&1
