timeout 1200 python -m pytest tests/test_gpu_f32.py tests/test_gpu_parity.py -x -q > gpurun_out/pytest_v4.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_v4.log
timeout 600 python exp/qt.py 2>&1 || true
