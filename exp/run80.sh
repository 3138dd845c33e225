timeout 900 python -m pytest tests/test_gpu_rs.py -x -q > gpurun_out/pytest_rs.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_rs.log
timeout 600 python bench.py --config rs-large --steps 10 --warmup 3 > gpurun_out/bench_rs_large.json 2> gpurun_out/bench_rs.err; echo b9=$?
timeout 600 python bench.py --config rs-small --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_rs_small.json 2>/dev/null; echo b10=$?
timeout 600 python bench.py --config rs-large --steps 3 --warmup 3 --no-sort --no-cpu-baseline > gpurun_out/bench_rs_large_unsorted.json 2>/dev/null; echo b12=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 100 --csv --log-file gpurun_out/launches_rs_large.csv python bench.py --config rs-large --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo ncu_launch_rs=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:k_rs_lookup -c 1 --csv --log-file gpurun_out/launch_rs_baseline.csv python tools/profile_rs.py --baseline --reps 0 > /dev/null 2>&1; echo ncu_base=$?
timeout 600 python bench.py > gpurun_out/bench_large.json 2> gpurun_out/bench_large.err; echo bench=$?
for f in gpurun_out/bench_rs_large.json gpurun_out/bench_large.json; do python -c "import json,sys;d=json.load(open('$f'));print(d['value'],d['ms_per_step'],d['roofline']['frac'],d['roofline'].get('traffic'),d['e2e']['value'],d['hash_matches_oracle'])"; done
