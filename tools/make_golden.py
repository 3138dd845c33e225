"""Write tests/golden/oracle_hashes.json: the oracle's verification sums for
the five BASELINE.json configs.  Calls only oracle/ (the stored values come
from the CPU oracle, never from the CUDA path).

    python tools/make_golden.py [--configs tiny,small,large,large-hash,xl] [--threads T]

Route: all three oracle routes give identical v (pin P9, tests/
test_oracle_rng_search.py), so each config uses the fastest route: the hash
route with the config's own bin count, or with many bins where the config
has no hash grid (a pure speed choice inside the oracle).
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
    "tiny": dict(I=12, N=1000, rule=1, L=100_000, bins=1024),
    "small": dict(I=68, N=11303, rule=0, L=17_000_000, bins=8192),
    "large": dict(I=355, N=11303, rule=0, L=17_000_000, bins=8192),
    "large-hash": dict(I=355, N=11303, rule=0, L=17_000_000, bins=8192),
    "xl": dict(I=355, N=238847, rule=0, L=170_000_000, bins=131072),
}
CONC_SEED = 1070 * 1070
HIST_PARTICLES, HIST_LOOKUPS = 500_000, 34   # XSBench history-mode defaults (R19)
HIST_PARTICLES_TINY = 3_000


def fnv1a(buf: bytes) -> str:
    h = 0xcbf29ce484222325
    for b in buf:
        h ^= b
        h = (h * 0x100000001b3) & 0xFFFFFFFFFFFFFFFF
    return f"{h:016x}"


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="tiny,small,large,large-hash,xl")
    ap.add_argument("--threads", type=int, default=os.cpu_count())
    ap.add_argument("--out", default=os.path.join(ROOT, "tests", "golden", "oracle_hashes.json"))
    ap.add_argument("--history-only", action="store_true",
                    help="only add the history-mode sums (R19: 500,000 particles x 34 "
                         "lookups, XSBench's history defaults) to existing entries")
    ap.add_argument("--f32-only", action="store_true",
                    help="only add the fp32-variant sums (R18) to existing entries")
    a = ap.parse_args()
    out = {}
    if os.path.exists(a.out):
        with open(a.out) as f:
            out = json.load(f)
    for name in a.configs.split(","):
        c = CONFIGS[name]
        t0 = time.time()
        o = oracle.Oracle.from_spec(c["I"], c["N"], grid_seed=42, conc_seed=CONC_SEED,
                                    material_rule=c["rule"], lookup_seed=1070,
                                    hash_bins=c["bins"], nthreads=a.threads)
        t1 = time.time()
        if a.history_only:
            P, L = (HIST_PARTICLES_TINY, 34) if name == "tiny" else (HIST_PARTICLES, HIST_LOOKUPS)
            Sh = o.run_history(0, P, L, mode=oracle.HASH, nthreads=a.threads)
            out[name]["history"] = dict(particles=P, lookups_per_particle=L, sum_v=int(Sh),
                                        hash=int(oracle.hash_finalize(Sh)))
            print(name, "history", P, L, Sh, flush=True)
            del o
            with open(a.out, "w") as f:
                json.dump(out, f, indent=1, sort_keys=True)
            continue
        if a.f32_only:
            S32 = o.run(0, c["L"], mode=oracle.HASH | oracle.F32, nthreads=a.threads)
            out[name]["sum_v_f32"] = int(S32)
            out[name]["hash_f32"] = int(oracle.hash_finalize(S32))
            print(name, "f32", S32, flush=True)
            del o
            with open(a.out, "w") as f:
                json.dump(out, f, indent=1, sort_keys=True)
            continue
        S = o.run(0, c["L"], mode=oracle.HASH, nthreads=a.threads)
        t2 = time.time()
        S32 = o.run(0, c["L"], mode=oracle.HASH | oracle.F32, nthreads=a.threads)
        # P11 regression fingerprints of the generated inputs (first 1 MiB of
        # the grid + the whole material tables)
        g = o.grid()
        entry = dict(n_isotopes=c["I"], n_gridpoints=c["N"], material_rule=c["rule"],
                     lookups=c["L"], grid_seed=42, conc_seed=CONC_SEED, lookup_seed=1070,
                     sum_v=int(S), hash=int(oracle.hash_finalize(S)),
                     sum_v_f32=int(S32), hash_f32=int(oracle.hash_finalize(S32)),
                     oracle_route=f"hash, {c['bins']} bins (P9: route-independent)",
                     fnv_grid_head=fnv1a(g.ravel()[:131072].tobytes()),
                     fnv_mats=fnv1a(o.mats().tobytes()), fnv_concs=fnv1a(o.concs().tobytes()),
                     grid_last=g[-1, -1].tolist(), oracle_seconds=round(t2 - t1, 1),
                     threads=a.threads, init_seconds=round(t1 - t0, 1))
        out[name] = entry
        print(name, entry, flush=True)
        del g, o
        with open(a.out, "w") as f:
            json.dump(out, f, indent=1, sort_keys=True)


if __name__ == "__main__":
    main()
