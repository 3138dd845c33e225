mkdir -p /tmp/reps
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_rs_lookup -s 1 -c 1 -o /tmp/reps/prof_rs python tools/profile_rs.py --lookups 2000000 > /dev/null 2>&1; echo ncu=$?
python tools/ncu_summary.py /tmp/reps/prof_rs.ncu-rep gpurun_out/ncu_rs_large 2000000 > /dev/null
python tools/ncu_mix.py /tmp/reps/prof_rs.ncu-rep 20 > gpurun_out/ncu_rs_large_mix.txt 2>&1
cp /tmp/reps/prof_rs.ncu-rep gpurun_out/prof_rs_large4.ncu-rep
