# fine pass: direct scatter for long segments (fine_direct sweep); colscan with 8 loads in flight
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "cbits or sorted or explicit or tiny" > gpurun_out/pytest_parity.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_parity.log
timeout 600 python exp/cbits.py large 0 10 0,1,2,1000 2>&1
timeout 900 python exp/cbits.py xl 0,8,9 3 0,2,1000 2>&1
timeout 600 python exp/cbits.py small 0 10 0,2,1000 2>&1
