"""Small invocations of every kernel family for compute-sanitizer's
racecheck / synccheck / initcheck (slow tools: tiny sizes only).

    compute-sanitizer --tool racecheck python tools/sanitize_tiny.py xs|rs
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_sc_tianscd23_b200.rs as RS  # noqa: E402
import paper_conf_sc_tianscd23_b200.xs as X  # noqa: E402

which = sys.argv[1]
if which == "xs":
    g = X.Grid.from_preset("tiny")
    L = 20_000
    for kw in ({}, {"sort": True}, {"sort": True, "f32": True}, {"baseline": True}):
        vs, _ = g.lookup(0, L, want=("macro_xs", "verification"), **kw)
        torch.cuda.synchronize()
        print("tiny", kw, vs.tolist(), flush=True)
    vs, _ = g.lookup(0, L, sort=True)   # vsum only (the bench launch: no positions)
    torch.cuda.synchronize()
    print("tiny sorted vsum-only", vs.tolist(), flush=True)
    for v in (20, 25):
        g.set_param("variant", v)
        vs, _ = g.lookup(0, L, sort=True, want=("macro_xs",))
        torch.cuda.synchronize()
        print("variant", v, vs.tolist(), flush=True)
    g.set_param("variant", 0)
    vs = torch.zeros(2, dtype=torch.int64, device="cuda")
    for r in range(3):
        g.lookup_shard(0, L, r, 3, vsum=vs)
    torch.cuda.synchronize()
    print("shards", vs.tolist(), flush=True)
    vs.zero_()   # 8 shards: lengthened tiles, one more coarse bit
    for r in range(8):
        g.lookup_shard(0, L, r, 8, vsum=vs)
    torch.cuda.synchronize()
    print("shards8", vs.tolist(), flush=True)
    vs, _ = g.lookup_history(0, 500, 4)
    torch.cuda.synchronize()
    print("history", vs.tolist(), flush=True)
    gh = X.Grid.from_preset("tiny", grid_type="hash", hash_bins=97)
    vs, _ = gh.lookup(0, L, sort=True)
    torch.cuda.synchronize()
    print("hash", vs.tolist(), flush=True)
else:
    p = RS.RSProblem.from_preset("rs-tiny")
    for kw in ({"sort": True}, {"sort": False}):
        vs, _ = p.lookup(0, 4_000, want=("macro_xs",), **kw)
        torch.cuda.synchronize()
        print("rs-tiny", kw, vs.tolist(), flush=True)
