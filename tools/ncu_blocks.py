"""Basic-block view of an ncu source page (SASS): consecutive instructions
with equal execution counts form a block; prints each hot block's
instructions per unit (e.g. per warp-nuclide step), stall-sample share and
opcode mix (development aid; DESIGN.md §4 uses it to split a kernel's
instructions into FP64 work and overhead).

  python tools/ncu_blocks.py SOURCE.csv|REPORT.ncu-rep UNITS [min_frac]
"""
import csv
import io
import subprocess
import sys
from collections import Counter


def rows_of(path):
    if path.endswith(".ncu-rep"):
        out = subprocess.run(["ncu", "-i", path, "--page", "source", "--csv", "--print-source",
                              "sass"], capture_output=True, text=True).stdout
        return list(csv.reader(io.StringIO(out)))
    return list(csv.reader(open(path)))


def main():
    rows = rows_of(sys.argv[1])
    units = float(sys.argv[2])
    thr = float(sys.argv[3]) if len(sys.argv) > 3 else 0.004
    # a multi-kernel export repeats "Kernel Name" / header rows: keep the first kernel
    hdr = rows[1]
    data = []
    for r in rows[2:]:
        if r and r[0] == "Kernel Name":
            break
        if r and r[0] != "Address":
            data.append(r)
    iA, iS = hdr.index("Address"), hdr.index("Source")
    iE, iW = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)")
    ins = [(int(r[iA], 16), r[iS].strip(), int(r[iE]), int(r[iW])) for r in data]
    base = ins[0][0]
    tot = sum(e for _, _, e, _ in ins)
    totw = sum(w for *_, w in ins) or 1
    fp_all = sum(e for _, s, e, _ in ins if s.lstrip("@!P0123456789T ").split(".")[0].split()[0]
                 in ("DMUL", "DADD", "DFMA"))
    print(f"instructions {tot} = {tot / units:.1f} per unit; FP64 {fp_all / units:.1f} per unit "
          f"({fp_all / tot:.3f})")
    blocks, cur = [], None
    for a, s, e, w in ins:
        op = (s.split()[1] if s.startswith("@") else s.split()[0]).split(".")[0]
        if cur and cur["e"] == e:
            cur["n"] += 1
            cur["w"] += w
            cur["ops"].append(op)
        else:
            cur = {"a": a - base, "e": e, "n": 1, "w": w, "ops": [op]}
            blocks.append(cur)
    for b in blocks:
        t = b["e"] * b["n"]
        if t > tot * thr:
            c = Counter(b["ops"])
            fp = sum(v for k, v in c.items() if k in ("DMUL", "DADD", "DFMA"))
            print(f"{b['a']:6x} exec {b['e']:9d} x {b['n']:4d} = {t / units:6.2f}/unit  "
                  f"samples {b['w'] / totw:.3f}  fp64 {fp:3d}  {dict(c.most_common(6))}")


if __name__ == "__main__":
    main()
