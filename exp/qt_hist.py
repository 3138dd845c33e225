import sys, torch
sys.path.insert(0, '.')
import paper_conf_sc_tianscd23_b200.xs as X
for cfg in sys.argv[1:] or ["large"]:
    g = X.Grid.from_preset(cfg)
    P, L = 500_000, 34
    for sort in [False, True]:
        vs = torch.zeros(2, dtype=torch.int64, device="cuda")
        g.lookup_history(0, P, L, sort=sort, vsum=vs); torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(3):
            vs.zero_(); g.lookup_history(0, P, L, sort=sort, vsum=vs)
        e1.record(); torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 3
        print(cfg, "history sort" if sort else "history", f"{ms:.3f} ms/step {P*L/ms/1e6:.3f} G lookups/s", vs.tolist(), X.hash_of(vs.cpu()), flush=True)
