import torch, time
n = 160 * 1024 * 1024
h = torch.empty(n, dtype=torch.uint8).pin_memory()
d = torch.empty(n, dtype=torch.uint8, device="cuda")
for ns in (1, 2, 4):
    streams = [torch.cuda.Stream() for _ in range(ns)]
    part = n // ns
    for rep in range(2):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(10):
            for k, s in enumerate(streams):
                with torch.cuda.stream(s):
                    d[k * part:(k + 1) * part].copy_(h[k * part:(k + 1) * part], non_blocking=True)
        torch.cuda.synchronize()
        dt = (time.perf_counter() - t0) / 10
    print(f"H2D {n >> 20} MiB over {ns} streams: {n / dt / 1e9:.1f} GB/s", flush=True)
# D2H too
torch.cuda.synchronize(); t0 = time.perf_counter()
for _ in range(10): h.copy_(d, non_blocking=True)
torch.cuda.synchronize(); print(f"D2H: {n * 10 / (time.perf_counter() - t0) / 1e9:.1f} GB/s")
