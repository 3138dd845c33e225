"""Dynamic SASS opcode mix + stall totals of an ncu report (development aid):
python tools/ncu_mix.py REPORT.ncu-rep [N]"""
import csv
import io
import subprocess
import sys
from collections import Counter

out = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "source", "--csv", "--print-source",
                      "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr, data = rows[1], rows[2:]
iS, iE = hdr.index("Source"), hdr.index("Instructions Executed")
cols = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
tot = {c: sum(int(r[hdr.index(c)] or 0) for r in data) for c in cols}
s = sum(tot.values()) or 1
print("stalls:", ", ".join(f"{c[6:]} {v / s:.3f}" for c, v in sorted(tot.items(), key=lambda x: -x[1])[:10]))
mix = Counter()
for r in data:
    t = r[iS].split()
    if not t:
        continue
    op = t[1] if t[0].startswith("@") else t[0]
    mix[op.split(".")[0]] += int(r[iE] or 0)
n = sum(mix.values())
print("instructions", n)
for k, v in mix.most_common(int(sys.argv[2]) if len(sys.argv) > 2 else 20):
    print(f"  {k:8s} {v:14d} {v / n:.3f}")
