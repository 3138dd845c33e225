timeout 900 python -m pytest tests/test_gpu_history.py -x -q > gpurun_out/pytest_hist.log 2>&1; echo pytest_hist=$?; tail -2 gpurun_out/pytest_hist.log
timeout 600 python bench.py --mode history --steps 10 > gpurun_out/bench_large_history.json 2>gpurun_out/bench_hist.err; echo b6=$?; cut -c1-250 gpurun_out/bench_large_history.json
