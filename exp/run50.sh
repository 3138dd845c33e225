timeout 600 python exp/rs_variants.py rs-large 0,1
timeout 600 python -m pytest tests/test_gpu_rs.py -x -q -k "tiny" 2>&1 | tail -2
