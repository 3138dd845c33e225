python - <<'PY'
import torch, time
x = torch.empty(204_000_000, dtype=torch.uint8).pin_memory()
y = torch.empty(204_000_000, dtype=torch.uint8, device="cuda")
for _ in range(3): y.copy_(x, non_blocking=True)
torch.cuda.synchronize()
e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(10): y.copy_(x, non_blocking=True)
e1.record(); torch.cuda.synchronize()
print("H2D pinned GB/s", 204e6 * 10 / (e0.elapsed_time(e1) / 1e3) / 1e9)
PY
python tools/e2e_sweep.py 17000000 8500000 5666667 4250000 2833334 2>&1 | tail -5
timeout 900 python bench.py --config xl --scaling strong --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_xl.json 2> gpurun_out/bench_xl.err; echo xl=$?; cut -c1-600 gpurun_out/bench_xl.json; tail -3 gpurun_out/bench_xl.err
