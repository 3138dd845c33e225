timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "tiny_full_parity or staged or ragged or layouts" > gpurun_out/pytest_v3.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_v3.log
for c in large large-hash small; do timeout 300 python tools/quick_time.py --config $c --variants sort-v19,sort-v21 2>&1 | tail -5; done
