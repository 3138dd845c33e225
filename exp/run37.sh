timeout 900 python -m pytest tests/test_gpu_rs.py -x -q > gpurun_out/pytest_rs.log 2>&1; echo pytest=$?; tail -30 gpurun_out/pytest_rs.log | grep -E "passed|failed|Error|assert|error" | head -20
timeout 600 python exp/rs_variants.py rs-large 0,3
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_rs_lookup -s 1 -c 1 -o gpurun_out/prof_rs_large3 python tools/profile_rs.py --lookups 2000000 > /dev/null 2>&1; echo ncu_full=$?
