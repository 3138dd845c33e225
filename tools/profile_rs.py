"""Run an RSBench config for ncu: one warm-up batch, then `--reps` more.
  ncu --set full -k regex:k_rs_lookup -s 1 -c 1 -o gpurun_out/prof_rs python tools/profile_rs.py
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_sc_tianscd23_b200.rs as RS  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="rs-large")
ap.add_argument("--reps", type=int, default=1)
ap.add_argument("--no-sort", action="store_true")
ap.add_argument("--baseline", action="store_true")
ap.add_argument("--lookups", type=int, default=0)
a = ap.parse_args()
p = RS.RSProblem.from_preset(a.config)
L = a.lookups or RS.RS_PRESETS[a.config]["lookups"]
vsum = torch.zeros(2, dtype=torch.int64, device="cuda")
for _ in range(1 + a.reps):
    p.lookup(0, L, sort=not a.no_sort, baseline=a.baseline, vsum=vsum)
torch.cuda.synchronize()
print([int(x) for x in vsum.cpu()])
