# ncu --set full of the XL gather (k_gather_s3, 170M sorted lookups)
mkdir -p gpurun_out /tmp/reps
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:k_gather_s3 -s 1 -c 1 -o /tmp/reps/prof_xl python tools/profile_one.py --config xl --lookups 170000000 --sort --reps 1 > gpurun_out/ncu_xl.log 2>&1; echo ncu=$?; tail -3 gpurun_out/ncu_xl.log
python tools/ncu_summary.py /tmp/reps/prof_xl.ncu-rep gpurun_out/ncu_gather_s3_xl 170000000 > /dev/null; echo sum=$?
python tools/ncu_regions.py /tmp/reps/prof_xl.ncu-rep > gpurun_out/ncu_gather_s3_xl_regions.txt 2>&1; echo reg=$?
python tools/ncu_mix.py /tmp/reps/prof_xl.ncu-rep 20 > gpurun_out/ncu_gather_s3_xl_mix.txt 2>&1
