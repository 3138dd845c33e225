"""Summarise an ncu --set full report (raw page) into a small JSON + text
table for profiles/.  Usage: python tools/ncu_summary.py REPORT.ncu-rep|RAW.csv OUT_PREFIX [LOOKUPS]"""
import csv
import io
import json
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
        "l1tex__t_sector_hit_rate.pct", "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum",
        "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum", "smsp__inst_executed.sum",
        "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "launch__occupancy_limit_registers",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed"]


def main():
    rep, out = sys.argv[1], sys.argv[2]
    lookups = int(sys.argv[3]) if len(sys.argv) > 3 else None
    if rep.endswith(".csv"):  # an exported `ncu -i ... --page raw --csv`
        raw = open(rep).read()
    else:
        raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                             text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        u = dict(zip(hdr, units))
        e = {"kernel": d.get("Kernel Name", "")[:80]}
        for k in KEYS:
            if k in d:
                try:
                    v = float(d[k].replace(",", ""))
                except ValueError:
                    continue
                unit = u.get(k, "")
                if unit in ("Gbyte",):
                    v *= 1e9
                elif unit in ("Mbyte",):
                    v *= 1e6
                elif unit in ("Kbyte",):
                    v *= 1e3
                elif unit == "msecond":
                    v *= 1e6
                elif unit == "usecond":
                    v *= 1e3
                e[k] = v
        if lookups and "dram__bytes_read.sum" in e:
            e["dram_bytes_per_lookup"] = (e["dram__bytes_read.sum"] +
                                          e.get("dram__bytes_write.sum", 0)) / lookups
        res.append(e)
    with open(out + ".json", "w") as f:
        json.dump(res, f, indent=1)
    with open(out + ".txt", "w") as f:
        for e in res:
            f.write(f"== {e['kernel']}\n")
            for k, v in e.items():
                if k != "kernel":
                    f.write(f"  {k:70s} {v:.6g}\n")
    print(open(out + ".txt").read())


if __name__ == "__main__":
    main()
