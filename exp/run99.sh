# final check of the committed state: full GPU tests, smoke, bench large/xl
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?; tail -1 gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench_large.json 2> gpurun_out/bench_large.err; echo bench=$?
timeout 900 python bench.py --config xl --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_xl.json 2>gpurun_out/bench_xl.err; echo xl=$?
timeout 600 python bench.py --config large-hash --no-cpu-baseline > gpurun_out/bench_large_hash.json 2>/dev/null; echo lh=$?
for f in large xl large_hash; do python -c "import json;d=json.load(open('gpurun_out/bench_$f.json'));print('$f',d['value'],d['ms_per_step'],d['roofline']['frac'],d.get('e2e',{}) and d['e2e'].get('value'),d.get('hash_matches_oracle'),d['gpu_launches'],d['clocks']['sm_mhz'],d['clocks']['reasons'])"; done
