timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "gate or explicit" > gpurun_out/pytest_gate2.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_gate2.log
timeout 900 python -m pytest tests/test_gpu_history.py -x -q > gpurun_out/pytest_hist.log 2>&1; echo pytest_hist=$?; tail -2 gpurun_out/pytest_hist.log
timeout 600 python bench.py --mode history --steps 10 > gpurun_out/bench_large_history.json 2>gpurun_out/bench_hist.err; echo b6=$?; cut -c1-250 gpurun_out/bench_large_history.json
timeout 600 python bench.py > gpurun_out/bench_large.json 2> gpurun_out/bench_large.err; echo bench=$?
python -c "import json;d=json.load(open('gpurun_out/bench_large.json'));print(d['value'],d['ms_per_step'],d['e2e']['value'],d['roofline']['frac'],d['gpu_launches'],d['hash_matches_oracle'],d['e2e']['vsum_matches_batch'])"
