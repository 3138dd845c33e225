# k_part_place reads the samples k_part_count kept (no second A1)
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_gpu.log
timeout 600 python exp/cbits.py large 0 10 2>&1
timeout 600 python exp/cbits.py small 0 10 2>&1
timeout 900 python exp/cbits.py xl 0 3 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_part" -c 10 --csv --log-file gpurun_out/launches_large_a2.csv python exp/cbits.py large 0 1 > /dev/null 2>&1; echo ncu=$?
