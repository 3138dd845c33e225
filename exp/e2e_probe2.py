import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sc_tianscd23_b200.xs as X
g = X.Grid.from_preset("large")
L = 17_000_000
_, res = g.lookup(0, L, sort=True, want=("energy", "mat"))
ed, md = res["energy"], res["mat"].to(torch.uint8)
vs = torch.zeros(2, dtype=torch.int64, device="cuda")
for name, f in (("batch", lambda: g.lookup(0, L, sort=True, vsum=vs)),
                ("explicit", lambda: g.lookup_explicit(ed, md, sort=True, vsum=vs))):
    f(); torch.cuda.synchronize()
    g.timing(True)
    for _ in range(5): f()
    torch.cuda.synchronize()
    t = g.timing_read(); g.timing(False)
    n = t["calls"]
    print(name, {k: round(t[k] / n, 3) for k in ("ms_count", "ms_bucket", "ms_gather")}, flush=True)
