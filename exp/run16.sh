timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -k "explicit" > gpurun_out/pytest_v5.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_v5.log
python tools/e2e_sweep.py 17000000 8500000 5666667 4250000 2>&1 | tail -4
