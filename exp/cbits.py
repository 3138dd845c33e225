"""Partitioned-A2 coarse-bit sweep (development aid): device time per step and
hash check for each part_cbits value (0 = by batch size)."""
import json, os, sys, time
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
import paper_conf_sc_tianscd23_b200.xs as X
cfg = sys.argv[1]
vals = [int(v) for v in sys.argv[2].split(",")]
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 5
fds = [int(v) for v in sys.argv[4].split(",")] if len(sys.argv) > 4 else [2]
variants = [int(v) for v in sys.argv[5].split(",")] if len(sys.argv) > 5 else [0]
caps = [int(v) for v in os.environ.get("FINE_CAPS", "0").split(",")]
gold = json.load(open(os.path.join(ROOT, "tests", "golden", "oracle_hashes.json")))
g = X.Grid.from_preset(cfg)
L = int(sys.argv[6]) if len(sys.argv) > 6 else X.PRESETS[cfg]["lookups"]
for c, fd, var, cap in [(c, fd, v, k) for c in vals for fd in fds for v in variants for k in caps]:
    g.set_param("fine_cap", cap)
    g.set_param("variant", var)
    g.set_param("part_cbits", c)
    g.set_param("fine_direct", fd)
    vsum = torch.zeros(2, dtype=torch.int64, device="cuda")
    g.lookup(0, L, vsum=vsum, sort=True)
    torch.cuda.synchronize()
    ok = int(vsum[0]) == gold[cfg]["sum_v"] if L == gold[cfg]["lookups"] else None
    g.timing(True)
    st = torch.cuda.Event(enable_timing=True); en = torch.cuda.Event(enable_timing=True)
    st.record()
    for _ in range(reps):
        vsum.zero_()
        g.lookup(0, L, vsum=vsum, sort=True)
    en.record(); torch.cuda.synchronize()
    ms = st.elapsed_time(en) / reps
    t = g.timing_read(); g.timing(False); n = t["calls"] or 1
    print(f"{cfg} cbits={c} fd={fd} v={var} cap={cap} {ms:8.3f} ms/step {L/ms/1e6:8.3f} G/s count {t['ms_count']/n:.3f} "
          f"bucket {t['ms_bucket']/n:.3f} gather {t['ms_gather']/n:.3f} hash_ok={ok}", flush=True)
