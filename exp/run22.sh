timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none -k regex:"k_part|k_gather" -c 12 --csv python tools/profile_one.py --config large --sort --reps 1 2>/dev/null | grep -v "^==" | awk -F'","' '{print $5, $13, $15}' | cut -c1-200
timeout 600 python exp/qt2.py large 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gather_s3 -s 1 -c 1 -o gpurun_out/prof_s3_large_b python tools/profile_one.py --config large --sort > gpurun_out/ncu_s3.log 2>&1; echo ncu_full=$?
