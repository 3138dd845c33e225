"""Write tests/golden/rs_oracle_sums.json: the RSBench oracle's verification
sums (R20-R27) for the rs-* workloads.  Calls only oracle/ (the
stored values come from the CPU oracle, never from the CUDA path).

    python tools/make_rs_golden.py [--configs rs-tiny,rs-small,rs-large] [--threads T]

Besides the whole-workload sum it stores the sums of fixed sub-ranges so a
GPU test can check a shard without the full workload.
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402

CONFIGS = {
    "rs-tiny": dict(I=12, rule=1, L=100_000),
    "rs-tiny-nodoppler": dict(I=12, rule=1, L=100_000, doppler=0),
    "rs-small": dict(I=68, rule=0, L=10_000_000),
    "rs-large": dict(I=355, rule=0, L=10_000_000),
}
SHARDS = [(0, 65_536), (1_000_003, 40_000)]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default=",".join(CONFIGS))
    ap.add_argument("--threads", type=int, default=os.cpu_count() or 1)
    a = ap.parse_args()
    path = os.path.join(ROOT, "tests", "golden", "rs_oracle_sums.json")
    out = json.load(open(path)) if os.path.exists(path) else {}
    for name in a.configs.split(","):
        c = CONFIGS[name]
        o = oracle.RSOracle(c["I"], 1000, 100, 4, c["rule"], 42, 1070, c.get("doppler", 1))
        t = time.time()
        S = o.run(0, c["L"], nthreads=a.threads)
        dt = time.time() - t
        shards = {f"{f}+{n}": o.run(f, n, nthreads=a.threads) for f, n in SHARDS if f + n <= c["L"]}
        out[name] = dict(n_nuclides=c["I"], material_rule=c["rule"], avg_n_poles=1000,
                         avg_n_windows=100, numL=4, doppler=c.get("doppler", 1), seed=42,
                         lookup_seed=1070, lookups=c["L"], sum_v=S,
                         hash=oracle.hash_finalize(S), shard_sums=shards,
                         oracle_seconds=round(dt, 1), oracle_threads=a.threads,
                         source="oracle/rs_oracle.c via tools/make_rs_golden.py")
        print(name, S, oracle.hash_finalize(S), f"{dt:.1f}s", flush=True)
        with open(path, "w") as f:
            json.dump(out, f, indent=1, sort_keys=True)


if __name__ == "__main__":
    main()
