import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, oracle
import paper_conf_sc_tianscd23_b200.rs as RS
for name, I, rule, L in (("rs-tiny", 12, 1, 100_000), ("rs-large", 355, 0, 20_000)):
    o = oracle.RSOracle(I, 1000, 100, material_rule=rule)
    S, ref = o.run(0, L, nthreads=os.cpu_count(), outputs=True)
    p = RS.RSProblem.from_spec(n_nuclides=I, material_rule=rule)
    vs, res = p.lookup(0, L, sort=True, want=("macro_xs",))
    torch.cuda.synchronize()
    M = res["macro_xs"].cpu().numpy()
    d = np.abs(M - ref["M"])
    print(name, "sum", int(vs[0]) == S, "max |dM|/(1+|M|) = %.3e" % (d / (1 + np.abs(ref["M"]))).max(),
          "max rel = %.3e" % (d / np.maximum(np.abs(ref["M"]), 1e-300)).max(),
          "median rel = %.3e" % np.median(d / np.maximum(np.abs(ref["M"]), 1e-300)),
          "bit-equal frac = %.4f" % np.mean(d == 0), flush=True)
