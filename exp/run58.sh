timeout 600 python exp/rs_variants.py rs-large 0
timeout 900 python -m pytest tests/test_gpu_rs.py -x -q > gpurun_out/pytest_rs.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_rs.log
