timeout 600 python tools/quick_time.py --config large --variants sort-v25 --reps 10
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "tiny or full_config" > gpurun_out/pytest_pick.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_pick.log
timeout 600 python exp/rs_variants.py rs-large 0
