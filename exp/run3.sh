timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "tiny_full_parity or staged" > gpurun_out/pytest_v2.log 2>&1; echo pytest=$?; tail -5 gpurun_out/pytest_v2.log
for c in large large-hash small; do timeout 300 python tools/quick_time.py --config $c --variants sort-v9,sort-v13,sort-v14,sort-v15,sort-v16 2>&1 | tail -6; done
