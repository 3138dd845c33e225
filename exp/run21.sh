timeout 600 python exp/qt2.py large 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_op_red.sum,lts__t_sectors_op_atom.sum --clock-control none -s 7 -c 7 --csv python tools/profile_one.py --config large --sort --reps 1 2>/dev/null | grep -v "^==" | cut -c1-250
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu.log
