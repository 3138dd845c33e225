timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_gather_s3 -s 1 -c 1 -o gpurun_out/gs3_large python tools/profile_one.py --config large --sort --reps 1 > gpurun_out/ncu_gs3.log 2>&1; echo ncu=$?
tail -2 gpurun_out/ncu_gs3.log
