timeout 900 python -m pytest tests/test_gpu_rs.py -x -q > gpurun_out/pytest_rs.log 2>&1; echo pytest=$?; tail -5 gpurun_out/pytest_rs.log | grep -E "passed|failed|Error|assert"
