# XL A2 launch list (ILP-4 fine pass)
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:k_part -c 10 --csv --log-file gpurun_out/launches_xl_a2.csv python exp/cbits.py xl 0 1 > /dev/null 2>&1; echo ncu=$?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:k_part -c 10 --csv --log-file gpurun_out/launches_large_a2.csv python exp/cbits.py large 0 1 > /dev/null 2>&1; echo ncu=$?
