timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_gather_s2 -s 1 -c 1 -o gpurun_out/gs2_large python tools/profile_one.py --config large --sort --reps 1 --variant 14 > gpurun_out/ncu_gs2.log 2>&1; echo ncu=$?
tail -3 gpurun_out/ncu_gs2.log
