python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench_large.json 2> gpurun_out/bench_large.err; echo bench=$?
cat gpurun_out/bench_large.json
timeout 600 python bench.py --config large-hash --no-cpu-baseline > gpurun_out/bench_large_hash.json 2>>gpurun_out/bench_large.err; echo bench=$?
timeout 600 python bench.py --config small --no-cpu-baseline > gpurun_out/bench_small.json 2>>gpurun_out/bench_large.err; echo bench=$?
timeout 600 python bench.py --no-sort --no-cpu-baseline --no-e2e > gpurun_out/bench_large_unsorted.json 2>>gpurun_out/bench_large.err; echo bench=$?
