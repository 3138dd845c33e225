import sys, torch
sys.path.insert(0, '.')
import paper_conf_sc_tianscd23_b200.xs as X
cfgs = sys.argv[1:] or ["large"]
for cfg in cfgs:
    g = X.Grid.from_preset(cfg)
    L = 17_000_000
    for f32, legacy in [(False, 1), (False, 0), (True, 0)]:
        g.set_param("legacy_sort", legacy)
        vs = torch.zeros(2, dtype=torch.int64, device="cuda")
        g.lookup(0, L, sort=True, vsum=vs, f32=f32); torch.cuda.synchronize()
        g.timing(True)
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(10):
            vs.zero_(); g.lookup(0, L, sort=True, vsum=vs, f32=f32)
        e1.record(); torch.cuda.synchronize()
        t = g.timing_read(); g.timing(False)
        ms = e0.elapsed_time(e1) / 10
        n = t['calls']
        print(cfg, "f32" if f32 else "f64", "legacy" if legacy else "part", f"{ms:.3f} ms/step {L/ms/1e6:.1f} M/s count {t['ms_count']/n:.3f} sort {t['ms_bucket']/n:.3f} gather {t['ms_gather']/n:.3f}", vs.tolist(), X.hash_of(vs.cpu()), flush=True)
    g.set_param("legacy_sort", 0)
    del g
