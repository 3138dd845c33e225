import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sc_tianscd23_b200.rs as RS
cfg = sys.argv[1] if len(sys.argv) > 1 else "rs-large"
gold = json.load(open("tests/golden/rs_oracle_sums.json"))[cfg]
p = RS.RSProblem.from_preset(cfg)
L = RS.RS_PRESETS[cfg]["lookups"]
vs = torch.zeros(2, dtype=torch.int64, device="cuda")
for v in [int(x) for x in (sys.argv[2].split(",") if len(sys.argv) > 2 else "0,1,2,3".split(","))]:
    p.set_param("variant", v)
    for sort in (True,):
        vs.zero_(); p.lookup(0, L, sort=sort, vsum=vs); torch.cuda.synchronize()
        ok = [int(x) for x in vs.cpu()] == [gold["sum_v"], L]
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(3):
            p.lookup(0, L, sort=sort, vsum=vs)
        e1.record(); torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 3
        print(f"variant {v} sort {sort}: {ms:.2f} ms  {L / ms / 1e3:.1f} M lookups/s  sum_ok {ok}", flush=True)
