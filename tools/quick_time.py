"""Quick per-variant device timing of one config (development aid; the
contract benchmark is bench.py).  Prints one line per variant."""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_sc_tianscd23_b200.xs as X  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="large")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--variants", default="v1,v2,v3,v4,sort,baseline")
    a = ap.parse_args()
    gold = json.load(open(os.path.join(ROOT, "tests", "golden", "oracle_hashes.json")))
    pre = dict(X.PRESETS[a.config])
    t0 = time.time()
    g = X.Grid.from_preset(a.config)
    torch.cuda.synchronize()
    print(f"init {a.config}: {time.time() - t0:.2f}s device_bytes={g.info.device_bytes/1e9:.2f}GB",
          flush=True)
    L = min(pre["lookups"], 17_000_000)
    for var in a.variants.split(","):
        kw = {}
        if var.startswith("v"):
            g.set_param("variant", int(var[1:]))
        if var.startswith("sort"):
            kw["sort"] = True
            if var != "sort":
                g.set_param("variant", int(var.split("-v")[-1]))
        if var == "baseline":
            kw["baseline"] = True
        for bps in [0]:
            g.set_param("blocks_per_sm", bps)
            vsum = torch.zeros(2, dtype=torch.int64, device="cuda")
            g.lookup(0, L, vsum=vsum, **kw)
            torch.cuda.synchronize()
            ok = int(vsum[0]) == gold[a.config]["sum_v"] if a.config in gold and L == gold[a.config]["lookups"] else None
            g.timing(True)
            st = torch.cuda.Event(enable_timing=True)
            en = torch.cuda.Event(enable_timing=True)
            st.record()
            for _ in range(a.reps):
                vsum.zero_()
                g.lookup(0, L, vsum=vsum, **kw)
            en.record()
            torch.cuda.synchronize()
            ms = st.elapsed_time(en) / a.reps
            t = g.timing_read()
            g.timing(False)
            n = t["calls"] or 1
            print(f"{var:9s} bps={bps} {ms:8.3f} ms/step  {L / ms / 1e6:8.3f} G lookups/s  "
                  f"count {t['ms_count']/n:.3f} bucket {t['ms_bucket']/n:.3f} gather {t['ms_gather']/n:.3f}"
                  f"  launches/step {t['kernel_launches']/n:.0f} hash_ok={ok}", flush=True)
        g.set_param("variant", 0)
        g.set_param("blocks_per_sm", 0)


if __name__ == "__main__":
    main()
