timeout 900 python -m pytest tests/test_gpu_rs.py -x -q > gpurun_out/pytest_rs.log 2>&1; echo pytest=$?; tail -15 gpurun_out/pytest_rs.log | grep -E "passed|failed|Error|assert" | head
timeout 600 python bench.py --config rs-large --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_rs_large_e2e.json 2> gpurun_out/bench_rs.err; echo b=$?; tail -3 gpurun_out/bench_rs.err
python -c "import json;d=json.load(open('gpurun_out/bench_rs_large_e2e.json'));print(d['value'],d['e2e'])"
