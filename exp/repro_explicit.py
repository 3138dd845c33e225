import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sc_tianscd23_b200.xs as X
cfg = sys.argv[1]
g = X.Grid.from_preset(cfg)
L = 17_000_000
vs0, res = g.lookup(0, L, sort=True, want=("energy", "mat"))
torch.cuda.synchronize()
print("batch", vs0.tolist(), flush=True)
e, m = res["energy"], res["mat"]
for n in [int(x) for x in sys.argv[2].split(",")]:
    for mode in sys.argv[3].split(","):
        try:
            if mode == "dev":
                vs, _ = g.lookup_explicit(e[:n], m[:n], sort=True)
            elif mode == "dev8":
                vs, _ = g.lookup_explicit(e[:n], m[:n].to(torch.uint8), sort=True)
            elif mode == "devns":
                vs, _ = g.lookup_explicit(e[:n], m[:n], sort=False)
            torch.cuda.synchronize()
            print(n, mode, vs.tolist(), flush=True)
        except Exception as ex:
            print(n, mode, "FAIL", ex, flush=True)
            sys.exit(1)
