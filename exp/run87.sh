# fine pass with 4 loads in flight per thread; colscan unrolled
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x > gpurun_out/pytest_parity.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_parity.log
timeout 600 python exp/cbits.py large 7,8,0 10 2>&1 | tee gpurun_out/cbits_large.txt
timeout 900 python exp/cbits.py xl 7,8,9,0 3 2>&1 | tee gpurun_out/cbits_xl.txt
timeout 600 python exp/cbits.py large-hash 0 10 2>&1
timeout 600 python exp/cbits.py small 0 10 2>&1
