"""Per-instruction view of an ncu report's source page (development aid):
python tools/ncu_src.py REPORT.ncu-rep [min_frac]  -> stall totals + hot SASS lines."""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
thr = float(sys.argv[2]) if len(sys.argv) > 2 else 0.0008
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr, data = rows[1], rows[2:]
iA, iS = hdr.index("Address"), hdr.index("Source")
iW, iE = hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Instructions Executed")
cols = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
tot = {c: sum(int(r[hdr.index(c)] or 0) for r in data) for c in cols}
s = sum(tot.values()) or 1
print("stalls:", ", ".join(f"{c[6:]} {v / s:.3f}" for c, v in sorted(tot.items(), key=lambda x: -x[1])[:9]))
te = sum(int(r[iE]) for r in data)
tw = sum(int(r[iW]) for r in data)
print("instructions executed", te, "samples", tw)
for r in data:
    e, w = int(r[iE]), int(r[iW])
    if e > te * thr or w > tw * 0.004:
        print(f"{r[iA][-5:]} {e:>10d} {w:>6d}  {r[iS].strip()[:80]}")
