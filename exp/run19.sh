# round-1 re-entry: confirm the restored tree on a fresh box
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench_large.json 2> gpurun_out/bench_large.err; echo bench=$?
cut -c1-400 gpurun_out/bench_large.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_large.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1; echo ncu_launch=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gather_s3 -s 1 -c 1 -o gpurun_out/prof_s3_large python tools/profile_one.py --config large --sort > gpurun_out/ncu_s3.log 2>&1; echo ncu_full=$?
timeout 900 ncu --set full --clock-control none -k regex:"k_sample|k_scatter" -s 2 -c 2 -o gpurun_out/prof_prep_large python tools/profile_one.py --config large --sort > gpurun_out/ncu_prep.log 2>&1; echo ncu_prep=$?
