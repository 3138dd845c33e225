timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "sub_batches or full_config" > gpurun_out/pytest_sub.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_sub.log
timeout 900 python bench.py --config xl --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_xl.json 2>gpurun_out/bench_xl.err; echo b8=$?; cut -c1-200 gpurun_out/bench_xl.json
python -c "import json;d=json.load(open('gpurun_out/bench_xl.json'));print(d['hash'],d['hash_matches_oracle'],d['phase_ms_per_step'],d['roofline']['frac'],d['gpu_launches'])"
