timeout 900 python -m pytest tests/test_gpu_history.py -x -q > gpurun_out/pytest_hist.log 2>&1; echo pytest=$?; tail -15 gpurun_out/pytest_hist.log
timeout 600 python exp/qt_hist.py large small 2>&1
timeout 600 python exp/qt3.py large 0 2>&1
