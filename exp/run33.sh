mkdir -p gpurun_out; nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -5 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?; tail -2 gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench_large.json 2> gpurun_out/bench_large.err; echo bench=$?
timeout 600 python bench.py --config small --no-cpu-baseline > gpurun_out/bench_small.json 2>/dev/null; echo b2=$?
timeout 600 python bench.py --config large-hash --no-cpu-baseline > gpurun_out/bench_large_hash.json 2>/dev/null; echo b3=$?
timeout 600 python bench.py --no-sort --no-cpu-baseline --steps 10 > gpurun_out/bench_large_unsorted.json 2>/dev/null; echo b4=$?
timeout 600 python bench.py --f32 --no-cpu-baseline > gpurun_out/bench_large_f32.json 2>/dev/null; echo b5=$?
timeout 600 python bench.py --mode history --steps 10 > gpurun_out/bench_large_history.json 2>gpurun_out/bench_hist.err; echo b6=$?
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_reference.json 2>/dev/null; echo b7=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_large.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1; echo ncu_launch=$?
mkdir -p /tmp/reps
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gather_s3 -s 1 -c 1 -o gpurun_out/prof_s3_large python tools/profile_one.py --config large --sort > /dev/null 2>&1; echo ncu_full=$?
timeout 900 ncu --set full --clock-control none -k regex:"k_part" -s 5 -c 5 -o /tmp/reps/prof_part_large python tools/profile_one.py --config large --sort > /dev/null 2>&1; echo ncu_part=$?
timeout 900 ncu --set full --clock-control none -k regex:"k_gather" -s 1 -c 1 -o /tmp/reps/prof_gather_unsorted python tools/profile_one.py --config large > /dev/null 2>&1; echo ncu_uns=$?
timeout 900 ncu --set full --clock-control none -k regex:"k_gather_s3" -s 1 -c 1 -o /tmp/reps/prof_s3_large_hash python tools/profile_one.py --config large-hash > /dev/null 2>&1; echo ncu_hash=$?
python tools/ncu_summary.py gpurun_out/prof_s3_large.ncu-rep gpurun_out/ncu_gather_s3_large 17000000 > /dev/null
python tools/ncu_summary.py /tmp/reps/prof_part_large.ncu-rep gpurun_out/ncu_part_large 17000000 > /dev/null
python tools/ncu_summary.py /tmp/reps/prof_gather_unsorted.ncu-rep gpurun_out/ncu_gather_large_unsorted 17000000 > /dev/null
python tools/ncu_summary.py /tmp/reps/prof_s3_large_hash.ncu-rep gpurun_out/ncu_gather_s3_large_hash 17000000 > /dev/null
python tools/ncu_regions.py gpurun_out/prof_s3_large.ncu-rep 64 > gpurun_out/ncu_gather_s3_regions.txt 2>&1
python tools/ncu_src.py gpurun_out/prof_s3_large.ncu-rep 0.004 > gpurun_out/ncu_gather_s3_source.txt 2>&1
ls -la gpurun_out
for f in gpurun_out/bench_*.json; do echo $f; cut -c1-200 $f; done
