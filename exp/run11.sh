ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_large.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/launches_bench.log 2>&1; echo launches=$?
mkdir -p /tmp/reps
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_gather_s3 -s 1 -c 1 -o /tmp/reps/gs3_large python tools/profile_one.py --config large --sort --reps 1 > /dev/null 2>&1; echo a=$?
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_gather_s3 -s 1 -c 1 -o /tmp/reps/gs3_large_hash python tools/profile_one.py --config large-hash --sort --reps 1 > /dev/null 2>&1; echo b=$?
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"k_sample|k_scatter|k_scan" -s 5 -c 5 -o /tmp/reps/prep_large python tools/profile_one.py --config large --sort --reps 1 > /dev/null 2>&1; echo c=$?
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"k_gather" -s 1 -c 1 -o /tmp/reps/g_large_unsorted python tools/profile_one.py --config large --reps 1 > /dev/null 2>&1; echo d=$?
python tools/ncu_summary.py /tmp/reps/gs3_large.ncu-rep gpurun_out/r01_ncu_gather_s3_large_sorted 17000000 > /dev/null
python tools/ncu_summary.py /tmp/reps/gs3_large_hash.ncu-rep gpurun_out/r01_ncu_gather_s3_large_hash 17000000 > /dev/null
python tools/ncu_summary.py /tmp/reps/prep_large.ncu-rep gpurun_out/r01_ncu_prep_large_sorted 17000000 > /dev/null
python tools/ncu_summary.py /tmp/reps/g_large_unsorted.ncu-rep gpurun_out/r01_ncu_gather_large_unsorted 17000000 > /dev/null
python tools/ncu_regions.py /tmp/reps/gs3_large.ncu-rep 48 > gpurun_out/r01_ncu_gather_s3_large_regions.txt
python tools/ncu_src.py /tmp/reps/gs3_large.ncu-rep 0.002 > gpurun_out/r01_ncu_gather_s3_large_source.txt
cp /tmp/reps/gs3_large.ncu-rep gpurun_out/
du -sh gpurun_out
