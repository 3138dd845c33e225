timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "host_io or explicit or full_config" > gpurun_out/pytest_fix.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_fix.log
timeout 600 python tools/e2e_sweep.py 17000000 8500000 4250000 2125000
