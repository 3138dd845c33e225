nvidia-smi --query-gpu=name,clocks.max.sm --format=csv,noheader
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench_large.json 2> gpurun_out/bench_large.err; echo bench=$?
timeout 600 python bench.py --config small --no-cpu-baseline > gpurun_out/bench_small.json 2>/dev/null; echo b2=$?
timeout 600 python bench.py --config large-hash --no-cpu-baseline > gpurun_out/bench_large_hash.json 2>/dev/null; echo b3=$?
timeout 600 python bench.py --no-sort --no-cpu-baseline --steps 10 > gpurun_out/bench_large_unsorted.json 2>/dev/null; echo b4=$?
timeout 600 python bench.py --f32 --no-cpu-baseline > gpurun_out/bench_large_f32.json 2>/dev/null; echo b5=$?
timeout 600 python bench.py --mode history --steps 10 > gpurun_out/bench_large_history.json 2>gpurun_out/bench_hist.err; echo b6=$?
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_reference.json 2>/dev/null; echo b7=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_large.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1; echo ncu_launch=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gather_s3 -s 1 -c 1 -o gpurun_out/prof_s3_large python tools/profile_one.py --config large --sort > gpurun_out/ncu_s3.log 2>&1; echo ncu_full=$?
timeout 900 ncu --set full --clock-control none -k regex:"k_part" -s 5 -c 5 -o gpurun_out/prof_part_large python tools/profile_one.py --config large --sort > gpurun_out/ncu_part.log 2>&1; echo ncu_part=$?
timeout 900 ncu --set full --clock-control none -k regex:"k_gather" -s 1 -c 1 -o gpurun_out/prof_gather_unsorted python tools/profile_one.py --config large > gpurun_out/ncu_uns.log 2>&1; echo ncu_uns=$?
for f in gpurun_out/bench_*.json; do echo $f; cut -c1-300 $f; done
