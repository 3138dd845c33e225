# partitioned-A2 coarse-bit sweep (large, XL) + the new parity tests
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -k cbits > gpurun_out/pytest_cbits.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_cbits.log
timeout 600 python exp/cbits.py large 7,8,9,0 10 2>&1 | tee gpurun_out/cbits_large.txt
timeout 900 python exp/cbits.py xl 7,8,9,0 3 2>&1 | tee gpurun_out/cbits_xl.txt
