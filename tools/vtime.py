"""Per-variant device timing of sorted batches (development aid; the
contract benchmark is bench.py).  One line per (variant, shard count):
step ms, phase ms (count / bucket / gather), vsum check against the golden
sum when the batch is the config's full batch.

  python tools/vtime.py --config large --variants 25,40,41 [--f32] [--shards 1,8]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_sc_tianscd23_b200.xs as X  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="large")
    ap.add_argument("--lookups", type=int, default=0)
    ap.add_argument("--variants", default="0")
    ap.add_argument("--shards", default="1")
    ap.add_argument("--f32", action="store_true")
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--index-layout", default="auto")
    ap.add_argument("--cbits", default="0", help="part_cbits values (comma list) tried per variant")
    ap.add_argument("--shard-tiles", default="0", help="shard_tiles values (comma list)")
    ap.add_argument("--fine-cap", default="0", help="fine_cap values (comma list)")
    a = ap.parse_args()
    gold = json.load(open(os.path.join(ROOT, "tests", "golden", "oracle_hashes.json")))[a.config]
    g = X.Grid.from_preset(a.config, index_layout=a.index_layout)
    L = a.lookups or X.PRESETS[a.config]["lookups"]
    st = torch.cuda.current_stream()
    for v, cb, stl, fc in [(int(x), int(c), int(t), int(f)) for x in a.variants.split(",")
                           for c in a.cbits.split(",") for t in a.shard_tiles.split(",")
                           for f in a.fine_cap.split(",")]:
        g.set_param("variant", v)
        g.set_param("part_cbits", cb)
        g.set_param("shard_tiles", stl)
        g.set_param("fine_cap", fc)
        for R in [int(x) for x in a.shards.split(",")]:
            worst, worst_ph, vs_tot = 0.0, None, [0, 0]
            for r in range(R):
                def run(vsum):
                    if R == 1:
                        g.lookup(0, L, sort=True, vsum=vsum, f32=a.f32)
                    else:
                        g.lookup_shard(0, L, r, R, vsum=vsum, f32=a.f32)
                vs = torch.zeros(2, dtype=torch.int64, device="cuda")
                run(vs)
                torch.cuda.synchronize()
                vs_tot = [vs_tot[0] + int(vs[0]), vs_tot[1] + int(vs[1])]
                for _ in range(2):
                    run(vs)
                g.timing(True)
                e0 = torch.cuda.Event(enable_timing=True)
                e1 = torch.cuda.Event(enable_timing=True)
                e0.record(st)
                for _ in range(a.reps):
                    run(vs)
                e1.record(st)
                torch.cuda.synchronize()
                ms = e0.elapsed_time(e1) / a.reps
                t = g.timing_read()
                g.timing(False)
                n = max(1, t["calls"])
                ph = (t["ms_count"] / n, t["ms_bucket"] / n, t["ms_gather"] / n)
                if ms > worst:
                    worst, worst_ph = ms, ph
            key = "sum_v_f32" if a.f32 else "sum_v"
            ok = vs_tot == [gold[key], L] if L == gold["lookups"] else None
            print(f"{a.config} L={L} f32={a.f32} variant={v} cbits={cb} stiles={stl} fcap={fc} shards={R}: step {worst:.4f} ms "
                  f"(count {worst_ph[0]:.4f} bucket {worst_ph[1]:.4f} gather {worst_ph[2]:.4f}) "
                  f"{L / worst / 1e6:.1f} M lookups/ms-equiv  vsum_ok={ok}", flush=True)


if __name__ == "__main__":
    main()
