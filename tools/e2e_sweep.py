"""Time the host-buffer explicit lookup (the bench's e2e leg) for several
host_chunk sizes (development aid)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_sc_tianscd23_b200.xs as X  # noqa: E402

g = X.Grid.from_preset("large")
L = 17_000_000
_, res = g.lookup(0, L, sort=True, want=("energy", "mat"))
e = res["energy"].cpu().pin_memory()
m = res["mat"].cpu().to(torch.uint8).pin_memory()
vs = torch.zeros(2, dtype=torch.int64).pin_memory()
for chunk in [int(a) for a in (sys.argv[1:] or ["17000000", "8500000", "4250000", "2125000"])]:
    g.set_param("host_chunk", chunk)
    g.lookup_explicit(e, m, sort=True, vsum=vs)
    t0 = time.perf_counter()
    for _ in range(5):
        vs.zero_()
        g.lookup_explicit(e, m, sort=True, vsum=vs)
    dt = (time.perf_counter() - t0) / 5
    print(f"chunk {chunk:>9d}: {dt*1e3:7.2f} ms  {L/dt/1e9:.3f} G lookups/s  vsum {vs.tolist()}",
          flush=True)
