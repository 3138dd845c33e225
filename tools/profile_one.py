"""Run a config for ncu: one warm-up lookup batch, then `--reps` more (the
profiled launches).  Usage under ncu:
  ncu --set full -k regex:k_gather -s 1 -c 1 -o gpurun_out/prof python tools/profile_one.py
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_sc_tianscd23_b200.xs as X  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="large")
ap.add_argument("--reps", type=int, default=2)
ap.add_argument("--sort", action="store_true")
ap.add_argument("--baseline", action="store_true")
ap.add_argument("--variant", type=int, default=0)
ap.add_argument("--lookups", type=int, default=0)
a = ap.parse_args()
g = X.Grid.from_preset(a.config)
if a.variant:
    g.set_param("variant", a.variant)
L = a.lookups or min(X.PRESETS[a.config]["lookups"], 17_000_000)
sort = a.sort or X.PRESETS[a.config].get("sort", False)
vsum = torch.zeros(2, dtype=torch.int64, device="cuda")
for _ in range(1 + a.reps):
    vsum.zero_()
    g.lookup(0, L, vsum=vsum, sort=sort, baseline=a.baseline)
torch.cuda.synchronize()
print("vsum", vsum.tolist(), "hash", X.hash_of(vsum.cpu()))
