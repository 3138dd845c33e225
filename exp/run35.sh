mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_rs.py -x -q > gpurun_out/pytest_rs.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_rs.log
timeout 600 python bench.py --config rs-large --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_rs_large.json 2> gpurun_out/bench_rs.err; echo bench=$?; tail -3 gpurun_out/bench_rs.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_rs_lookup -s 1 -c 1 -o gpurun_out/prof_rs_large2 python tools/profile_rs.py --lookups 2000000 > /dev/null 2>&1; echo ncu_full=$?
python tools/ncu_summary.py gpurun_out/prof_rs_large2.ncu-rep gpurun_out/ncu_rs_large2 2000000 > /dev/null 2>&1
cut -c1-300 gpurun_out/bench_rs_large.json
