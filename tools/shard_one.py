"""Run shard r of R of the sampled batch (for ncu): warm-up + `--reps`."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_sc_tianscd23_b200.xs as X  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="large")
ap.add_argument("--shard", type=int, default=0)
ap.add_argument("--shards", type=int, default=8)
ap.add_argument("--reps", type=int, default=1)
ap.add_argument("--variant", type=int, default=0)
a = ap.parse_args()
g = X.Grid.from_preset(a.config)
g.set_param("variant", a.variant)
L = X.PRESETS[a.config]["lookups"]
vs = torch.zeros(2, dtype=torch.int64, device="cuda")
for _ in range(1 + a.reps):
    g.lookup_shard(0, L, a.shard, a.shards, vsum=vs)
torch.cuda.synchronize()
print("vsum", vs.tolist())
