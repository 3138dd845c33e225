timeout 600 python tools/quick_time.py --config large --variants sort-v25 --reps 10
timeout 600 python tools/quick_time.py --config large-hash --variants sort-v25 --reps 10
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_f32.py -x -q > gpurun_out/pytest_fine.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_fine.log
