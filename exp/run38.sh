mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --config rs-large --steps 10 --warmup 3 > gpurun_out/bench_rs_large.json 2> gpurun_out/bench_rs.err; echo bench=$?; tail -3 gpurun_out/bench_rs.err
timeout 600 python bench.py --config rs-small --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_rs_small.json 2>/dev/null; echo b2=$?
timeout 600 python bench.py --config rs-large --steps 3 --warmup 3 --no-sort --no-cpu-baseline > gpurun_out/bench_rs_large_nosort.json 2>/dev/null; echo b3=$?
timeout 600 python bench.py --config rs-large --impl reference --steps 3 --warmup 3 > gpurun_out/bench_rs_reference.json 2>/dev/null; echo b4=$?
timeout 300 python tools/profile_rs.py --baseline --lookups 10000000 > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 100 --csv --log-file gpurun_out/launches_rs_large.csv python bench.py --config rs-large --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo ncu_launch=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:k_rs_lookup -c 1 --csv --log-file gpurun_out/launch_rs_baseline.csv python tools/profile_rs.py --baseline --reps 0 > /dev/null 2>&1; echo ncu_base=$?
for f in gpurun_out/bench_rs*.json; do echo $f; cut -c1-400 $f; done
