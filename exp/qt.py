import sys, torch, time
sys.path.insert(0, '.')
import paper_conf_sc_tianscd23_b200.xs as X
for cfg in ["large", "small", "large-hash"]:
    g = X.Grid.from_preset(cfg)
    L = 17_000_000
    for f32, var in [(False, 0), (True, 0), (True, 36)]:
        g.set_param("variant", var)
        vs = torch.zeros(2, dtype=torch.int64, device="cuda")
        g.lookup(0, L, sort=True, vsum=vs, f32=f32); torch.cuda.synchronize()
        g.timing(True)
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(5):
            vs.zero_(); g.lookup(0, L, sort=True, vsum=vs, f32=f32)
        e1.record(); torch.cuda.synchronize()
        t = g.timing_read(); g.timing(False)
        ms = e0.elapsed_time(e1) / 5
        n = t['calls']
        print(cfg, "f32" if f32 else "f64", var, f"{ms:.3f} ms/step {L/ms/1e6:.3f} G/s sample {t['ms_count']/n:.3f} scan+scatter {t['ms_bucket']/n:.3f} gather {t['ms_gather']/n:.3f}", vs.tolist(), flush=True)
    g.set_param("variant", 0)
    del g
