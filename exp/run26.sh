timeout 600 python exp/qt3.py large 0 2>&1
timeout 600 python exp/qt3.py large-hash 0 2>&1
timeout 600 python exp/qt3.py small 0 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_f32.py -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gather_s3 -s 1 -c 1 -o gpurun_out/prof_s3_large_c python tools/profile_one.py --config large --sort > gpurun_out/ncu_s3.log 2>&1; echo ncu_full=$?
