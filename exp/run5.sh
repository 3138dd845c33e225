timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "tiny_full_parity or staged" > gpurun_out/pytest_v3.log 2>&1; echo pytest=$?; tail -5 gpurun_out/pytest_v3.log
for c in large large-hash small; do timeout 300 python tools/quick_time.py --config $c --variants sort-v9,sort-v14,sort-v17,sort-v18,sort-v19,sort-v20 2>&1 | tail -7; done
