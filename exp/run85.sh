# full verification of the checkpointed state: GPU tests, smoke, default bench, reference arm
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke.log 2>&1; echo smoke=$?; tail -2 gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench_large.json 2> gpurun_out/bench_large.err; echo bench=$?
timeout 600 python bench.py --impl reference > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err; echo ref=$?
timeout 600 python bench.py --config rs-large --steps 10 --warmup 3 > gpurun_out/bench_rs_large.json 2> gpurun_out/bench_rs.err; echo b9=$?
for f in gpurun_out/bench_rs_large.json gpurun_out/bench_large.json; do python -c "import json,sys;d=json.load(open('$f'));print(d['value'],d['ms_per_step'],d['roofline']['frac'],d['roofline'].get('traffic'),d['e2e']['value'],d.get('hash_matches_oracle'),d['clocks'])"; done
cat gpurun_out/bench_reference.json
