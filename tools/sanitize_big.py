import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sc_tianscd23_b200.xs as X
import paper_conf_sc_tianscd23_b200.rs as RS
g = X.Grid.from_preset("large")
for kw in ({"sort": True}, {"sort": True, "f32": True}):
    vs, _ = g.lookup(0, 17_000_000, **kw)
    torch.cuda.synchronize()
    print("large", kw, vs.tolist(), flush=True)
g.close()
p = RS.RSProblem.from_preset("rs-large")
vs, _ = p.lookup(0, 1_000_000, sort=True, want=("macro_xs",))
torch.cuda.synchronize()
print("rs-large 1M", vs.tolist(), flush=True)
