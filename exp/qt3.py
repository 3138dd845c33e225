import sys, torch
sys.path.insert(0, '.')
import paper_conf_sc_tianscd23_b200.xs as X
cfg = sys.argv[1]
variants = [int(v) for v in sys.argv[2:]]
g = X.Grid.from_preset(cfg)
L = 17_000_000
for var in variants:
    g.set_param("variant", var)
    vs = torch.zeros(2, dtype=torch.int64, device="cuda")
    g.lookup(0, L, sort=True, vsum=vs); torch.cuda.synchronize()
    g.timing(True)
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(10):
        vs.zero_(); g.lookup(0, L, sort=True, vsum=vs)
    e1.record(); torch.cuda.synchronize()
    t = g.timing_read(); g.timing(False)
    ms = e0.elapsed_time(e1) / 10
    n = t['calls']
    print(cfg, var, f"{ms:.3f} ms/step {L/ms/1e6:.1f} M/s count {t['ms_count']/n:.3f} sort {t['ms_bucket']/n:.3f} gather {t['ms_gather']/n:.3f}", X.hash_of(vs.cpu()), flush=True)
