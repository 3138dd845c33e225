timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "above_48m or host_io or ragged or vsum_only" > gpurun_out/pytest_48m.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_48m.log
