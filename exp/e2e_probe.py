import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sc_tianscd23_b200.xs as X
g = X.Grid.from_preset("large")
L = 17_000_000
_, res = g.lookup(0, L, sort=True, want=("energy", "mat"))
ed, md = res["energy"], res["mat"].to(torch.uint8)
e, m = ed.cpu().pin_memory(), md.cpu().pin_memory()
torch.cuda.synchronize()
def timeit(f, n=5):
    f(); torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(n): f()
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) / n * 1e3
d1 = torch.empty_like(ed); d2 = torch.empty_like(md)
print("H2D only      %.2f ms" % timeit(lambda: (d1.copy_(e, non_blocking=True), d2.copy_(m, non_blocking=True))))
vs = torch.zeros(2, dtype=torch.int64, device="cuda")
print("device explicit %.2f ms" % timeit(lambda: g.lookup_explicit(ed, md, sort=True, vsum=vs)))
print("device batch  %.2f ms" % timeit(lambda: g.lookup(0, L, sort=True, vsum=vs)))
vh = torch.zeros(2, dtype=torch.int64).pin_memory()
for ch in (17_000_000, 8_500_000, 5_666_667, 4_250_000, 2_833_334):
    g.set_param("host_chunk", ch)
    print("host explicit chunk %d: %.2f ms" % (ch, timeit(lambda: g.lookup_explicit(e, m, sort=True, vsum=vh))))
