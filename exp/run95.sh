# density-based staged-gather choice: full GPU tests, smoke, bench lines
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?; tail -1 gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench_large.json 2> gpurun_out/bench_large.err; echo bench=$?
timeout 900 python bench.py --config xl --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_xl.json 2>gpurun_out/bench_xl.err; echo xl=$?
timeout 600 python bench.py --config small --no-cpu-baseline > gpurun_out/bench_small.json 2>/dev/null; echo small=$?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_part|k_gather_s3" -c 6 --csv --log-file gpurun_out/launches_xl.csv python bench.py --config xl --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1; echo ncu_xl=$?
for f in large xl small; do python -c "import json;d=json.load(open('gpurun_out/bench_$f.json'));print('$f',d['value'],d['ms_per_step'],d['roofline']['frac'],d.get('e2e',{}) and d['e2e'].get('value'),d.get('hash_matches_oracle'),d.get('phase_ms_per_step'),d['clocks']['sm_mhz'],d['clocks']['reasons'])"; done
