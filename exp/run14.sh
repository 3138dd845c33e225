mkdir -p /tmp/reps
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_gather_s3 -s 1 -c 1 -o /tmp/reps/gs3_large python tools/profile_one.py --config large --sort --reps 1 > /dev/null 2>&1; echo a=$?
python tools/ncu_summary.py /tmp/reps/gs3_large.ncu-rep gpurun_out/cur_gs3 17000000 > /dev/null
python tools/ncu_regions.py /tmp/reps/gs3_large.ncu-rep 32 > gpurun_out/cur_gs3_regions.txt
python tools/ncu_src.py /tmp/reps/gs3_large.ncu-rep 0.001 > gpurun_out/cur_gs3_source.txt
cp /tmp/reps/gs3_large.ncu-rep gpurun_out/cur_gs3.ncu-rep
