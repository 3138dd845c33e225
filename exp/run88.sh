# fine pass with 8 loads in flight per thread
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "cbits or sorted or explicit" > gpurun_out/pytest_parity.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_parity.log
timeout 600 python exp/cbits.py large 0 10 2>&1
timeout 900 python exp/cbits.py xl 0 3 2>&1
timeout 600 python exp/cbits.py small 0 10 2>&1
