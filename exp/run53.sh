mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu,power.draw --format=csv > gpurun_out/gpu.txt
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?; tail -2 gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench_large.json 2> gpurun_out/bench_large.err; echo bench=$?
timeout 600 python bench.py --config small --no-cpu-baseline > gpurun_out/bench_small.json 2>/dev/null; echo b2=$?
timeout 600 python bench.py --config large-hash --no-cpu-baseline > gpurun_out/bench_large_hash.json 2>/dev/null; echo b3=$?
timeout 600 python bench.py --no-sort --no-cpu-baseline --steps 10 > gpurun_out/bench_large_unsorted.json 2>/dev/null; echo b4=$?
timeout 600 python bench.py --f32 --no-cpu-baseline > gpurun_out/bench_large_f32.json 2>/dev/null; echo b5=$?
timeout 600 python bench.py --mode history --steps 10 > gpurun_out/bench_large_history.json 2>gpurun_out/bench_hist.err; echo b6=$?
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_reference.json 2>/dev/null; echo b7=$?
timeout 900 python bench.py --config xl --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_xl.json 2>gpurun_out/bench_xl.err; echo b8=$?
timeout 600 python bench.py --config rs-large --steps 10 --warmup 3 > gpurun_out/bench_rs_large.json 2> gpurun_out/bench_rs.err; echo b9=$?
timeout 600 python bench.py --config rs-small --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_rs_small.json 2>/dev/null; echo b10=$?
timeout 600 python bench.py --config rs-large --impl reference --steps 3 --warmup 3 > gpurun_out/bench_rs_reference.json 2>/dev/null; echo b11=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_large.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1; echo ncu_launch=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 100 --csv --log-file gpurun_out/launches_rs_large.csv python bench.py --config rs-large --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo ncu_launch_rs=$?
mkdir -p /tmp/reps
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gather_s3 -s 1 -c 1 -o /tmp/reps/prof_s3_large python tools/profile_one.py --config large --sort > /dev/null 2>&1; echo ncu_full=$?
timeout 900 ncu --set full --clock-control none -k regex:"k_part" -s 5 -c 5 -o /tmp/reps/prof_part_large python tools/profile_one.py --config large --sort > /dev/null 2>&1; echo ncu_part=$?
timeout 900 ncu --set full --clock-control none -k regex:k_gather_s3 -s 1 -c 1 -o /tmp/reps/prof_s3_small python tools/profile_one.py --config small --sort > /dev/null 2>&1; echo ncu_small=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_rs_lookup -s 1 -c 1 -o /tmp/reps/prof_rs_large python tools/profile_rs.py --lookups 2000000 > /dev/null 2>&1; echo ncu_rs=$?
python tools/ncu_summary.py /tmp/reps/prof_s3_large.ncu-rep gpurun_out/ncu_gather_s3_large 17000000 > /dev/null
python tools/ncu_summary.py /tmp/reps/prof_part_large.ncu-rep gpurun_out/ncu_part_large 17000000 > /dev/null
python tools/ncu_summary.py /tmp/reps/prof_s3_small.ncu-rep gpurun_out/ncu_gather_s3_small 17000000 > /dev/null
python tools/ncu_summary.py /tmp/reps/prof_rs_large.ncu-rep gpurun_out/ncu_rs_large 2000000 > /dev/null
python tools/ncu_mix.py /tmp/reps/prof_rs_large.ncu-rep 20 > gpurun_out/ncu_rs_large_mix.txt 2>&1
python tools/ncu_mix.py /tmp/reps/prof_s3_large.ncu-rep 20 > gpurun_out/ncu_gather_s3_large_mix.txt 2>&1
python tools/ncu_regions.py /tmp/reps/prof_s3_large.ncu-rep 64 > gpurun_out/ncu_gather_s3_regions.txt 2>&1
for f in gpurun_out/bench_*.json; do echo $f; cut -c1-220 $f; done
