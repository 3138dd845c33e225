"""Stall-sample and instruction shares of consecutive SASS regions of an ncu
report (development aid): python tools/ncu_regions.py REPORT [lines_per_region]"""
import csv
import io
import subprocess
import sys

out = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "source", "--csv", "--print-source",
                      "sass"], capture_output=True, text=True).stdout
n = int(sys.argv[2]) if len(sys.argv) > 2 else 64
rows = list(csv.reader(io.StringIO(out)))
hdr, data = rows[1], rows[2:]
iA, iS = hdr.index("Address"), hdr.index("Source")
iW, iE = hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Instructions Executed")
tw = sum(int(r[iW]) for r in data)
te = sum(int(r[iE]) for r in data)
acc = acce = 0
first = data[0][iA]
for i, r in enumerate(data):
    acc += int(r[iW])
    acce += int(r[iE])
    if (i + 1) % n == 0 or i == len(data) - 1:
        if acc or acce:
            print(f"{first[-5:]}-{r[iA][-5:]} samples {acc / tw:6.3f} inst {acce / te:6.3f}  "
                  f"{r[iS].strip()[:40]}")
        acc = acce = 0
        if i + 1 < len(data):
            first = data[i + 1][iA]
