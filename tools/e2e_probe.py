"""H2D bandwidth and the host-input lookup call at several chunk sizes
(development aid for the e2e leg)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_sc_tianscd23_b200.xs as X  # noqa: E402

n = 153_000_000
h = torch.empty(n, dtype=torch.uint8).pin_memory()
d = torch.empty(n, dtype=torch.uint8, device="cuda")
for _ in range(3):
    d.copy_(h, non_blocking=True)
torch.cuda.synchronize()
t0 = time.perf_counter()
for _ in range(10):
    d.copy_(h, non_blocking=True)
torch.cuda.synchronize()
dt = (time.perf_counter() - t0) / 10
print(f"H2D pinned {n / dt / 1e9:.1f} GB/s ({dt * 1e3:.2f} ms for 153 MB)", flush=True)
g = X.Grid.from_preset("large")
L = 17_000_000
_, r = g.lookup(0, L, sort=True, want=("energy", "mat"))
e = r["energy"].cpu().pin_memory()
m = r["mat"].cpu().to(torch.uint8).pin_memory()
vs = torch.zeros(2, dtype=torch.int64).pin_memory()
for chunk in [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else
                                "17000000,8500000,5666667,4250000,3400000").split(",")]:
    g.set_param("host_chunk", chunk)
    for _ in range(2):
        g.lookup_explicit(e, m, sort=True, vsum=vs)
    t0 = time.perf_counter()
    for _ in range(5):
        vs.zero_()
        g.lookup_explicit(e, m, sort=True, vsum=vs)
    dt = (time.perf_counter() - t0) / 5
    print(f"host_chunk {chunk}: {dt * 1e3:.2f} ms per call, {L / dt / 1e9:.2f} G lookups/s, "
          f"vsum {vs.tolist()}", flush=True)
