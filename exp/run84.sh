timeout 600 python bench.py --config rs-large --steps 10 --warmup 3 > gpurun_out/bench_rs_large.json 2> gpurun_out/bench_rs.err; echo b9=$?
timeout 600 python bench.py --config rs-small --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_rs_small.json 2>/dev/null; echo b10=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 100 --csv --log-file gpurun_out/launches_rs_large.csv python bench.py --config rs-large --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo ncu_launch_rs=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:k_rs_lookup -c 1 --csv --log-file gpurun_out/launch_rs_baseline.csv python tools/profile_rs.py --baseline --reps 0 > /dev/null 2>&1; echo ncu_base=$?
bash exp/run73.sh
python -c "import json;d=json.load(open('gpurun_out/bench_rs_large.json'));print(d['value'],d['ms_per_step'],d['roofline']['frac'],d['e2e']['value'],d['hash_matches_oracle'],d['cpu_baseline']['value'])"
