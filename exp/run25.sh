timeout 600 python exp/qt3.py large 0 2>&1
timeout 600 python exp/qt2.py large-hash small 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_f32.py -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu.log
