timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_part|k_gather_s3" -c 6 --csv --log-file gpurun_out/launches_xl.csv python bench.py --config xl --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1; echo ncu=$?
grep -v "^==" gpurun_out/launches_xl.csv | awk -F'","' '{print $5, $NF}' | cut -c1-120
