set -x
./tools/fp64_peak > gpurun_out/fp64_peak.json; cat gpurun_out/fp64_peak.json
nvidia-smi --query-gpu=clocks.sm --format=csv
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_gather_s -s 1 -c 1 -o gpurun_out/gs_large python tools/profile_one.py --config large --sort --reps 1 > gpurun_out/ncu_gs.log 2>&1; echo ncu=$?
tail -3 gpurun_out/ncu_gs.log
