import sys; sys.path.insert(0,'.')
import numpy as np, torch, oracle
import paper_conf_sc_tianscd23_b200.xs as X
g = X.Grid.from_preset("tiny")
o = oracle.Oracle.from_spec(12, 1000, conc_seed=1070*1070, material_rule=1)
S, ref = o.run(0, 100000, nthreads=8, outputs=True)
vs, res = g.lookup(0, 100000, want=("macro_xs","energy","mat","grid_index","verification"))
torch.cuda.synchronize()
out = {k: v.cpu().numpy() for k,v in res.items()}
for k, rk in (("energy","p"),("mat","mat"),("grid_index","grid_index"),("verification","v")):
    bad = np.nonzero(out[k] != ref[rk])[0]
    print(k, len(bad), bad[:10], out[k][bad[:5]], ref[rk][bad[:5]])
bad = np.nonzero(~np.all(out["macro_xs"]==ref["M"],axis=1))[0]
print("M", len(bad), bad[:10])
print(vs.tolist(), S)
