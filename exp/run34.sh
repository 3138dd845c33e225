mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_rs.py -x -q > gpurun_out/pytest_rs.log 2>&1; echo pytest=$?; tail -15 gpurun_out/pytest_rs.log
timeout 600 python bench.py --config rs-large --steps 5 --warmup 3 > gpurun_out/bench_rs_large.json 2> gpurun_out/bench_rs.err; echo bench=$?; tail -3 gpurun_out/bench_rs.err
timeout 600 python bench.py --config rs-large --steps 3 --warmup 3 --no-sort --no-cpu-baseline > gpurun_out/bench_rs_large_nosort.json 2>/dev/null; echo b2=$?
timeout 300 python tools/profile_rs.py --baseline --lookups 2000000 > gpurun_out/rs_baseline.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 100 --csv --log-file gpurun_out/launches_rs_large.csv python bench.py --config rs-large --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo ncu_launch=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_rs_lookup -s 1 -c 1 -o gpurun_out/prof_rs_large python tools/profile_rs.py --lookups 2000000 > /dev/null 2>&1; echo ncu_full=$?
python tools/ncu_summary.py gpurun_out/prof_rs_large.ncu-rep gpurun_out/ncu_rs_large 2000000 > /dev/null 2>&1
for f in gpurun_out/bench_rs*.json; do echo $f; cut -c1-600 $f; done
