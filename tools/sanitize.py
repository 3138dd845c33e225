"""Run the main entry points once each at modest sizes (for compute-sanitizer)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sc_tianscd23_b200.xs as X
import paper_conf_sc_tianscd23_b200.rs as RS
which = sys.argv[1]
if which == "xs":
    for cfg, L in (("tiny", 100_000), ("small", 1_000_000)):
        g = X.Grid.from_preset(cfg)
        for kw in ({}, {"sort": True}, {"baseline": True}, {"sort": True, "f32": True}):
            vs, res = g.lookup(0, L, want=("macro_xs", "energy", "mat", "verification"), **kw)
            torch.cuda.synchronize()
            print(cfg, kw, vs.tolist(), flush=True)
        vs, res = g.lookup(0, L, sort=True, want=("energy", "mat"))
        e, m = res["energy"].cpu().pin_memory(), res["mat"].cpu().to(torch.uint8).pin_memory()
        vs2 = torch.zeros(2, dtype=torch.int64).pin_memory()
        g.lookup_explicit(e, m, sort=True, vsum=vs2)
        print(cfg, "host explicit", vs2.tolist(), flush=True)
        vs3, _ = g.lookup_history(0, 2000, 34)
        torch.cuda.synchronize()
        print(cfg, "history", vs3.tolist(), flush=True)
        g.close()
    gh = X.Grid.from_preset("tiny", grid_type="hash", hash_bins=97)
    vs, _ = gh.lookup(0, 100_000, sort=True); torch.cuda.synchronize(); print("hash", vs.tolist())
else:
    for cfg, L in (("rs-tiny", 50_000), ("rs-small", 200_000)):
        p = RS.RSProblem.from_preset(cfg)
        for kw in ({"sort": True}, {"sort": False}, {"baseline": True}):
            vs, res = p.lookup(0, L, want=("macro_xs", "mat", "energy"), **kw)
            torch.cuda.synchronize()
            print(cfg, kw, vs.tolist(), flush=True)
        print(cfg, "work", p.work_count(0, L), flush=True)
        p.close()
