#!/usr/bin/env python
"""bench.py — XSBench event-based macroscopic XS lookups/s on B200.

Metric (BASELINE.json): XS lookups/sec at 1/2/4/8 B200 and the fraction of
the HBM-gather roofline.  One step = one pass of the whole hot path (A1
sample, A2 (material, energy) binning, A3 unionized/hash search, A4-A8
gather, interpolate, accumulate, verify; A9 all-reduce when N > 1) over one
batch of synthetic lookups whose tables are resident in HBM.  At N = 1 the
workload is XSBench "large" (355 nuclides x 11,303 points, 17M lookups,
unionized grid) — the configuration BASELINE.json's target is quoted on.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config large]
                  [--impl ours|reference] [--scaling weak|strong] [--no-sort]
  (N > 1: python -m torch.distributed.run --nproc-per-node N ... bench.py --gpus N)

--impl reference times the CPU oracle (oracle/, plain serial C per lookup)
on the host cores, as the reference arm of this tier.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

ORACLE_MODE = {"unionized": 0, "nuclide": 1, "hash": 2}
MAT_PROB = [0.139, .052, .275, .134, .154, .064, .066, .055, .008, .015, .025, .013]


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default="large",
                    choices=["tiny", "small", "large", "large-hash", "xl", "rs-tiny", "rs-small",
                             "rs-large"])
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--scaling", default="strong", choices=["weak", "strong"],
                    help="strong (default): L lookups in total over N GPUs; weak: L per GPU")
    ap.add_argument("--shard", default="energy", choices=["energy", "ids"],
                    help="strong scaling of sorted batches: energy-range shards of all L "
                         "lookups (default) or contiguous id ranges")
    ap.add_argument("--no-extras", action="store_true",
                    help="skip the N=1 context legs (strong-scaling projection, unsorted "
                         "batch, the paper's kernel shape)")
    ap.add_argument("--extra-steps", type=int, default=10)
    ap.add_argument("--no-sort", action="store_true", help="skip A2 (material/energy binning)")
    ap.add_argument("--f32", action="store_true",
                    help="the fp32 variant (XS_FLAG_F32, DESIGN.md R18; hash vs the oracle's "
                         "fp32 golden sum)")
    ap.add_argument("--lookups", type=int, default=0, help="override lookups per GPU (weak)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=20)
    ap.add_argument("--backend", default="nccl", choices=["nccl", "gloo"],
                    help="process-group backend (gloo: host-side A9, for single-GPU testing "
                         "of the multi-rank path; ranks then share GPUs round-robin)")
    ap.add_argument("--cpu-seconds", type=float, default=12.0,
                    help="target CPU seconds of the oracle sample")
    ap.add_argument("--mode", default="event", choices=["event", "history"],
                    help="event (default; the paper's XSBench -m event) or history "
                         "(DESIGN.md R19: particles x chained lookups)")
    ap.add_argument("--particles", type=int, default=500_000,
                    help="history mode: particles per GPU (weak) / in total (strong)")
    ap.add_argument("--lookups-per-particle", type=int, default=34)
    return ap.parse_args()


# ----------------------------------------------------------------- clocks --
class ClockSampler:
    """Samples SM clock and throttle reasons with NVML during the timed region."""

    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
               0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
               0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown",
               0x100: "display_clock_setting"}

    def __init__(self, index: int, period: float = 0.02):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self.period = period
        self._stop = threading.Event()
        self._t = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self._nv = pynvml
            self._h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self._h, pynvml.NVML_CLOCK_SM)
        except Exception as e:  # pragma: no cover - NVML missing
            self._nv = None
            self.error = str(e)

    def _run(self):
        nv = self._nv
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self._h, nv.NVML_CLOCK_SM))
                r = nv.nvmlDeviceGetCurrentClocksEventReasons(self._h)
                for bit, name in self.REASONS.items():
                    if r & bit and name != "gpu_idle":
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        if self._nv:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._t:
            self._t.join()

    def summary(self):
        if not self._nv:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvml_unavailable"]}
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons),
                "samples": len(self.samples)}


# ------------------------------------------------------------- helpers ------
def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


GATHER_KERNEL = {True: "k_gather_s4 (A4-A8, cp.async-staged interval-table windows)",
                 False: "k_gather_u (A4-A8, 3 lanes x 256-bit loads per lookup)"}
FP64_OPS_PER_LOOKUP_NUCLIDE = 24
FP64_OPS_F32_VARIANT = 5
FP64_LANES_PER_SM = 64   # B200: 37 TFLOP/s FP64 (FMA = 2) = 148 SMs x 64 lanes x 2 x 1.965 GHz


def fp64_pipe_peak():
    """FP64 pipe peak in T ops/s: 148 SMs x 64 FP64 lanes x max SM clock
    (tools/fp64_peak.cu measures 63.8 DADD/DMUL per SM per clock)."""
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    mhz, src = 1965.0, "derived: 148 SMs x 64 FP64 lanes x 1965 MHz (B200 max SM clock)"
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        if d.get("sm_max_mhz"):
            mhz = float(d["sm_max_mhz"])
            src = (f"derived: 148 SMs x 64 FP64 lanes x {mhz:.0f} MHz (MEASURED_PEAKS.json "
                   "sm_max_mhz); measured 18.55 T DADD/s (profiles/fp64_peak.json)")
    return 148 * FP64_LANES_PER_SM * mhz * 1e6 / 1e12, src


def golden():
    with open(os.path.join(ROOT, "tests", "golden", "oracle_hashes.json")) as f:
        return json.load(f)


def ncu_traffic(config: str, sort: bool):
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if not os.path.exists(p):
        return None, None
    with open(p) as f:
        d = json.load(f)
    e = d.get(f"{config}{'-sorted' if sort else ''}")
    if not e:
        return None, None
    return e.get("dram_bytes_per_lookup"), e.get("source")


def cpu_info():
    name = None
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    name = line.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    return name


def oracle_sample_rate(pre, target_s: float, first: int = 0, f32: bool = False,
                       cores: int | None = None):
    """Time the CPU oracle (as it stands) on a bounded sample of the workload
    on all host cores (or `cores` threads).  Returns (lookups/s, cores,
    description, sum_v, n)."""
    import oracle
    cores = cores or os.cpu_count() or 1
    mode = ORACLE_MODE[pre["grid_type"]] | (oracle.F32 if f32 else 0)
    o = oracle.Oracle.from_spec(pre["n_isotopes"], pre["n_gridpoints"], conc_seed=1070 * 1070,
                                material_rule=pre["material_rule"],
                                hash_bins=pre.get("hash_bins", 0), nthreads=cores)
    pilot = min(pre["lookups"], 20_000)
    t0 = time.perf_counter()
    o.run(first, pilot, mode=mode, nthreads=cores)
    dt = max(time.perf_counter() - t0, 1e-6)
    n = int(min(pre["lookups"], max(pilot, pilot / dt * target_s)))
    t0 = time.perf_counter()
    S = o.run(first, n, mode=mode, nthreads=cores)
    dt = time.perf_counter() - t0
    desc = (f"lookup ids [{first}, {first + n}) of the {pre['lookups']:,}-lookup "
            f"{pre['grid_type']} workload, oracle route '{pre['grid_type']}', {cores} threads, "
            f"{dt:.1f} s")
    return n / dt, cores, desc, S, n


# ------------------------------------------------------------- reference ----
def run_reference(a, pre, cfg):
    rank = int(os.environ.get("RANK", 0))
    if rank != 0:
        return 0
    t_start = time.time()
    # size each step to a bounded sample so the whole run takes a few minutes
    budget = 150.0
    per_step = max(1.0, min(a.cpu_seconds, budget / max(1, a.steps + a.warmup)))
    rate0, cores, _, _, _ = oracle_sample_rate(pre, per_step / 4, f32=a.f32)
    n = int(min(pre["lookups"], max(10_000, rate0 * per_step)))
    import oracle
    mode = ORACLE_MODE[pre["grid_type"]] | (oracle.F32 if a.f32 else 0)
    o = oracle.Oracle.from_spec(pre["n_isotopes"], pre["n_gridpoints"], conc_seed=1070 * 1070,
                                material_rule=pre["material_rule"],
                                hash_bins=pre.get("hash_bins", 0), nthreads=cores)
    for w in range(a.warmup):
        o.run((w * n) % max(1, pre["lookups"] - n + 1), n, mode=mode, nthreads=cores)
    times = []
    for k in range(a.steps):
        first = (k * n) % max(1, pre["lookups"] - n + 1)
        t0 = time.perf_counter()
        o.run(first, n, mode=mode, nthreads=cores)
        times.append(time.perf_counter() - t0)
    tot = sum(times)
    value = n * a.steps / tot
    line = {"impl": "reference", "metric": "XS lookups/sec", "value": value,
            "unit": "lookups/s", "n_gpus": a.gpus, "steps": a.steps, "warmup": a.warmup,
            "ms_per_step": 1e3 * tot / a.steps, "higher_is_better": True,
            "scaling": a.scaling, "vs_baseline": None, "dtype": "f32" if a.f32 else "f64",
            "data": "synthetic",
            "config": cfg,
            "cpu_baseline": {"value": value, "unit": "lookups/s", "cores": cores,
                             "kind": "oracle",
                             "sample": f"{n:,} lookups per step ({pre['grid_type']} route), "
                                       f"{cores} host threads, {cpu_info()}"},
            "e2e": {"value": value, "unit": "lookups/s", "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0},
            "wall_s": round(time.time() - t_start, 1)}
    print(json.dumps(line), flush=True)
    return 0


# ----------------------------------------------------------- history mode --
def run_history(a, pre, cfg):
    """History mode (R19): one step = all chained lookups of this
    rank's particles (lookups_per_particle rounds of the event pipeline)."""
    import torch
    import torch.distributed as dist

    from paper_conf_sc_tianscd23_b200 import dist as D
    from paper_conf_sc_tianscd23_b200 import xs as X

    rank, world, local = D.env_rank()
    local = local % torch.cuda.device_count()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl" if a.backend == "nccl" else "gloo",
                                **({"device_id": dev} if a.backend == "nccl" else {}))
    Lp = a.lookups_per_particle
    first, n = D.shard_range(rank, world, a.particles, a.scaling)
    # each round is a batch of n independent lookups at random energies: the
    # material-bucketed gather beats per-round energy binning there (measured:
    # large 1.14 vs 0.27 G lookups/s), so history rounds skip A2
    sort = False
    t0 = time.time()
    g = X.Grid.from_preset(a.config, device=local)
    torch.cuda.synchronize()
    init_s = time.time() - t0
    stream = torch.cuda.current_stream(dev)
    vsum = torch.zeros(2, dtype=torch.int64, device=dev)

    def step():
        vsum.zero_()
        g.lookup_history(first, n, Lp, sort=sort, vsum=vsum)
        if world > 1:
            if a.backend == "nccl":
                D.combine_vsum(vsum)
            else:
                vsum.copy_(D.combine_vsum(vsum.cpu()))

    for _ in range(a.warmup):
        step()
    torch.cuda.synchronize()
    g.timing(True)
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        ev0.record(stream)
        for _ in range(a.steps):
            step()
        ev1.record(stream)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
    ms_local = ev0.elapsed_time(ev1)
    tm = g.timing_read()
    g.timing(False)
    ms = D.max_over_ranks(ms_local, device=dev if a.backend == "nccl" else None)
    total = (n * world if a.scaling == "weak" else a.particles) * Lp * a.steps
    value = total / (ms / 1e3)
    vglob = [int(x) for x in vsum.cpu()]
    gold = golden().get(a.config, {}).get("history")
    hash_check = None
    if gold and world == 1 and first == 0 and n == gold["particles"] and \
            Lp == gold["lookups_per_particle"]:
        hash_check = vglob == [gold["sum_v"], n * Lp]
    # whole-step roofline against HBM: every round is an unsorted-or-binned
    # gather of n lookups; algorithmic bytes = sum over chained lookups of
    # n_nuclides(mat) x (4 + 96) B (E[n] from the material distribution)
    num_nucs = g.table(X.XS_TABLE_NUM_NUCS).tolist()
    en = sum(p * k for p, k in zip(MAT_PROB, num_nucs))
    balg = en * 100 + (8 * math.ceil(math.log2(max(2, g.info.n_union - 1)))
                       if pre["grid_type"] == "unionized" else 0)
    peak, peak_src = measured_peaks()
    achieved = balg * value / world / 1e9
    line = {"metric": "XS lookups/sec", "mode": "history", "value": value,
            "unit": "lookups/s", "n_gpus": world, "steps": a.steps, "warmup": a.warmup,
            "ms_per_step": ms / a.steps, "higher_is_better": True, "scaling": a.scaling,
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": dict(cfg, mode="history", particles_per_gpu=n,
                           lookups_per_particle=Lp,
                           sort="material buckets per round (no energy binning)"),
            "roofline": {"bound": "hbm", "kernel": "whole step (lookups_per_particle rounds)",
                         "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": None, "peak_source": peak_src,
                         "note": f"algorithmic bytes per chained lookup = {balg:.0f} "
                                 "(E[n] x (4 + 96) B + unionized search probes)"},
            "gpu_launches": int(tm["kernel_launches"]),
            "hash": D.global_hash(vglob), "lookups_per_step": vglob[1],
            "hash_matches_oracle": hash_check, "init_s": round(init_s, 2),
            "clocks": clk.summary()}
    # e2e: the public call from a host program (nothing to upload: particles
    # are generated on the device), vsum read back every step
    vs_h = torch.zeros(2, dtype=torch.int64).pin_memory()
    t0 = time.perf_counter()
    for _ in range(a.e2e_steps):
        step()
        vs_h.copy_(vsum)
    dt = time.perf_counter() - t0
    dt = D.max_over_ranks(dt, device=dev if a.backend == "nccl" else None)
    line["e2e"] = {"value": (n * world if a.scaling == "weak" else a.particles) * Lp *
                   a.e2e_steps / dt, "unit": "lookups/s", "h2d_bytes_per_step": 0,
                   "d2h_bytes_per_step": 16,
                   "api": "xs_lookup_history + vsum D2H, wall clock", "steps": a.e2e_steps}
    if rank == 0 and world == 1 and not a.no_cpu_baseline:
        import oracle
        cores = os.cpu_count() or 1
        o = oracle.Oracle.from_spec(pre["n_isotopes"], pre["n_gridpoints"],
                                    conc_seed=1070 * 1070, material_rule=pre["material_rule"],
                                    hash_bins=pre.get("hash_bins", 0), nthreads=cores)
        mode = ORACLE_MODE[pre["grid_type"]]
        pilot = 500
        t0 = time.perf_counter()
        o.run_history(0, pilot, Lp, mode=mode, nthreads=cores)
        rate = pilot / max(time.perf_counter() - t0, 1e-6)
        m = int(min(n, max(pilot, rate * a.cpu_seconds)))
        t0 = time.perf_counter()
        o.run_history(0, m, Lp, mode=mode, nthreads=cores)
        dt = time.perf_counter() - t0
        line["cpu_baseline"] = {"value": m * Lp / dt, "unit": "lookups/s", "cores": cores,
                                "kind": "oracle",
                                "sample": f"particles [0, {m}) x {Lp} chained lookups, oracle "
                                          f"route '{pre['grid_type']}', {cores} threads, "
                                          f"{dt:.1f} s", "cpu": cpu_info()}
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


# ---------------------------------------------------------------- RSBench --
# FP64 operations of the multipole lookup as the kernels evaluate it (DESIGN.md
# §10): each add/sub/mul/fma/compare instruction is one (products and sums
# contract into FMAs, R28); a complex division by a shared denominator is 3
# for the reciprocal's Newton step + 1 per quotient (in the series the a_n
# weight is folded into the reciprocal: 1 product for both quotients); sqrt, sin, cos and IEEE
# division count ONE each (so frac is a lower bound on the pipe time the
# transcendentals really take).  Per pole: the FP64 instructions of the
# compiled pole loop (ncu source view, profiles/r01_ncu_rs_lookup_large_mix.txt).
RS_OPS_PER_POLE = 152
RS_OPS_PER_NUCLIDE = 91
RS_OPS_PER_LOOKUP = 11


def rs_cpu_rate(pre, target_s, first=0):
    import oracle
    cores = os.cpu_count() or 1
    o = oracle.RSOracle(pre["n_nuclides"], 1000, 100, 4, pre["material_rule"], 42, 1070, 1)
    pilot = min(pre["lookups"], 2000)
    t0 = time.perf_counter()
    o.run(first, pilot, nthreads=cores)
    dt = max(time.perf_counter() - t0, 1e-6)
    n = int(min(pre["lookups"], max(pilot, pilot / dt * target_s)))
    t0 = time.perf_counter()
    S = o.run(first, n, nthreads=cores)
    dt = time.perf_counter() - t0
    return n / dt, cores, n, dt, S


def run_rs(a, pre, cfg):
    """RSBench event mode: one step = R1-R7 over this
    rank's lookups, vsum all-reduced for N > 1."""
    import torch
    import torch.distributed as dist

    from paper_conf_sc_tianscd23_b200 import dist as D
    from paper_conf_sc_tianscd23_b200 import rs as RS

    rank, world, local = D.env_rank()
    if a.impl == "reference":
        if rank != 0:
            return 0
        budget = 150.0
        per_step = max(1.0, min(a.cpu_seconds, budget / max(1, a.steps + a.warmup)))
        rate0, cores, n, _, _ = rs_cpu_rate(pre, per_step / 4)
        n = int(min(pre["lookups"], max(1000, rate0 * per_step)))
        import oracle
        o = oracle.RSOracle(pre["n_nuclides"], 1000, 100, 4, pre["material_rule"], 42, 1070, 1)
        for w in range(a.warmup):
            o.run(w * n, n, nthreads=cores)
        times = []
        for k in range(a.steps):
            t0 = time.perf_counter()
            o.run((k * n) % max(1, pre["lookups"] - n + 1), n, nthreads=cores)
            times.append(time.perf_counter() - t0)
        value = n * a.steps / sum(times)
        print(json.dumps({"impl": "reference", "metric": "RS lookups/sec", "value": value,
                          "unit": "lookups/s", "n_gpus": a.gpus, "steps": a.steps,
                          "warmup": a.warmup, "ms_per_step": 1e3 * sum(times) / a.steps,
                          "higher_is_better": True, "scaling": a.scaling, "vs_baseline": None,
                          "dtype": "f64", "data": "synthetic", "config": cfg,
                          "cpu_baseline": {"value": value, "unit": "lookups/s", "cores": cores,
                                           "kind": "oracle",
                                           "sample": f"{n:,} lookups per step, {cores} host "
                                                     f"threads, {cpu_info()}"},
                          "e2e": {"value": value, "unit": "lookups/s", "h2d_bytes_per_step": 0,
                                  "d2h_bytes_per_step": 0}}), flush=True)
        return 0
    local = local % torch.cuda.device_count()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl" if a.backend == "nccl" else "gloo",
                                **({"device_id": dev} if a.backend == "nccl" else {}))
    sort = not a.no_sort
    L_cfg = a.lookups or pre["lookups"]
    first, L = D.shard_range(rank, world, L_cfg, a.scaling)
    t0 = time.time()
    p = RS.RSProblem.from_spec(device=local, **pre)
    torch.cuda.synchronize()
    init_s = time.time() - t0
    stream = torch.cuda.current_stream(dev)
    n_nuc, n_pole = p.work_count(first, L)
    vsum = torch.zeros(2, dtype=torch.int64, device=dev)

    def step():
        vsum.zero_()
        p.lookup(first, L, sort=sort, vsum=vsum)
        if world > 1:
            if a.backend == "nccl":
                D.combine_vsum(vsum)
            else:
                vsum.copy_(D.combine_vsum(vsum.cpu()))

    for _ in range(a.warmup):
        step()
    torch.cuda.synchronize()
    l0 = p.launches
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        ev0.record(stream)
        for _ in range(a.steps):
            step()
        ev1.record(stream)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
    ms_local = ev0.elapsed_time(ev1)
    launches = p.launches - l0
    ms = D.max_over_ranks(ms_local, device=dev if a.backend == "nccl" else None)
    total = L * world * a.steps if a.scaling == "weak" else L_cfg * a.steps
    value = total / (ms / 1e3)
    vglob = [int(x) for x in vsum.cpu()]
    # the lookup kernel's own time (sample/bucket kernels excluded), events on the stream
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    ws = p.workspace(L, RS.RS_FLAG_SORT if sort else 0)
    vs2 = torch.zeros(2, dtype=torch.int64, device=dev)
    e0.record(stream)
    for _ in range(3):
        p.lookup(first, L, sort=sort, vsum=vs2)
    e1.record(stream)
    torch.cuda.synchronize()
    step_ms_lookup = e0.elapsed_time(e1) / 3
    del ws
    ops = n_pole * RS_OPS_PER_POLE + n_nuc * RS_OPS_PER_NUCLIDE + L * RS_OPS_PER_LOOKUP
    peak, peak_src = fp64_pipe_peak()
    achieved = ops / (ms_local / a.steps / 1e3) / 1e12
    with open(os.path.join(ROOT, "tests", "golden", "rs_oracle_sums.json")) as f:
        gold = json.load(f).get(a.config)
    hash_check = None
    if gold and world == 1 and first == 0 and L == gold["lookups"]:
        hash_check = vglob == [gold["sum_v"], L]
    line = {"metric": "RS lookups/sec", "app": "rsbench", "value": value, "unit": "lookups/s",
            "n_gpus": world, "steps": a.steps, "warmup": a.warmup,
            "ms_per_step": ms / a.steps, "higher_is_better": True, "scaling": a.scaling,
            "vs_baseline": None, "dtype": "f64", "data": "synthetic", "config": cfg,
            "roofline": {"bound": "alu", "kernel": "whole step (k_rs_lookup dominant)",
                         "achieved": achieved, "peak": peak, "unit": "TFLOP/s",
                         "frac": achieved / peak, "traffic": None, "peak_source": peak_src,
                         "algorithmic_fp64_ops_per_step": ops,
                         "units": {"lookup_nuclide": n_nuc, "pole_terms": n_pole},
                         "note": f"{RS_OPS_PER_POLE} FP64 ops per pole term, "
                                 f"{RS_OPS_PER_NUCLIDE} per (lookup, nuclide), "
                                 f"{RS_OPS_PER_LOOKUP} per lookup; sqrt/sin/cos/IEEE "
                                 "division count one each (DESIGN.md §10)"},
            "gpu_launches": int(launches),
            "hash": D.global_hash(vglob), "lookups_per_step": vglob[1],
            "hash_matches_oracle": hash_check, "init_s": round(init_s, 2),
            "device_bytes": int(p.device_bytes), "step_ms_recheck": step_ms_lookup}
    # e2e: the shard's (energy, material) pairs from pinned host memory through
    # rs_lookup_explicit(RS_FLAG_HOST_IO): H2D of 9 B per lookup, the lookups,
    # vsum back to the host, inside the timed call
    _, r0 = p.lookup(first, L, sort=sort, want=("energy", "mat"))
    e_host = r0["energy"].cpu().pin_memory()
    m_host = r0["mat"].cpu().to(torch.uint8).pin_memory()
    del r0
    vs_h = torch.zeros(2, dtype=torch.int64).pin_memory()
    p.lookup_explicit(e_host, m_host, sort=sort, vsum=vs_h)   # warm-up
    if world > 1:
        dist.barrier()
    t0 = time.perf_counter()
    for _ in range(a.e2e_steps):
        vs_h.zero_()
        p.lookup_explicit(e_host, m_host, sort=sort, vsum=vs_h)
    dt = D.max_over_ranks(time.perf_counter() - t0, device=dev if a.backend == "nccl" else None)
    line["e2e"] = {"value": (L * world if a.scaling == "weak" else L_cfg) * a.e2e_steps / dt,
                   "unit": "lookups/s", "h2d_bytes_per_step": int(L * 9),
                   "d2h_bytes_per_step": 16,
                   "api": "rs_lookup_explicit(RS_FLAG_HOST_IO): pinned host energy (f64) + "
                          "material (u8) in, vsum out; wall clock per call (the call "
                          "synchronizes)", "steps": a.e2e_steps,
                   "vsum_matches_batch": [int(x) for x in vs_h] == [int(x) for x in vsum.cpu()]}
    line["clocks"] = clk.summary()
    if rank == 0 and world == 1 and not a.no_cpu_baseline:
        rate, cores, n, dt, _ = rs_cpu_rate(pre, a.cpu_seconds)
        line["cpu_baseline"] = {"value": rate, "unit": "lookups/s", "cores": cores,
                                "kind": "oracle",
                                "sample": f"lookup ids [0, {n}) of {pre['lookups']:,}, "
                                          f"{cores} threads, {dt:.1f} s", "cpu": cpu_info()}
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


# ------------------------------------------------------------------ ours ----
def _timed_steps(step, stream, k, world, dist):
    """k steps bracketed by barrier + synchronize, one CUDA event per step
    boundary on the launching stream.  Returns (total ms, per-step ms list)."""
    import torch
    evs = [torch.cuda.Event(enable_timing=True) for _ in range(k + 1)]
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    evs[0].record(stream)
    for q in range(k):
        step()
        evs[q + 1].record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    per = [evs[q].elapsed_time(evs[q + 1]) for q in range(k)]
    return evs[0].elapsed_time(evs[k]), per


def _time_fn(fn, stream, k, warm=2):
    import torch
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(k):
        fn()
    e1.record(stream)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / k


def strong_projection(g, L, f32, stream, value1, ms1, steps=5, passes=2):
    """One-GPU projection of strong scaling (L fixed): every rank's shard is
    timed alone on this GPU; the R-GPU step is the slowest shard (the A9
    all-reduce of 16 bytes, ~20 us over NVLink, is not included).  Two
    partitions: energy-range shards (the bench's multi-GPU default,
    xs_lookup_batch_shard) and contiguous id ranges.  A shard's time is the
    lower of `passes` means over `steps` steps, so that a transient on the
    one shared GPU (a clock dip while one shard is timed) does not stand in
    for that rank's step."""
    out = {}
    for R in (2, 4, 8):
        per_e, per_i = [], []
        for r in range(R):
            per_e.append(min(_time_fn(lambda: g.lookup_shard(0, L, r, R, f32=f32), stream, steps)
                             for _ in range(passes)))
            a, b = r * L // R, (r + 1) * L // R
            per_i.append(min(_time_fn(lambda: g.lookup(a, b - a, sort=True, f32=f32), stream, steps)
                             for _ in range(passes)))
        me, mi = max(per_e), max(per_i)
        out[str(R)] = {"energy_shards": {"ms_per_step": me, "value": L / (me / 1e3),
                                         "speedup": ms1 / me, "efficiency": ms1 / me / R,
                                         "rank_ms": [round(x, 4) for x in per_e]},
                       "id_shards": {"ms_per_step": mi, "value": L / (mi / 1e3),
                                     "speedup": ms1 / mi, "efficiency": ms1 / mi / R}}
    return out


def run_ours(a, pre, cfg):
    import torch
    import torch.distributed as dist

    from paper_conf_sc_tianscd23_b200 import dist as D
    from paper_conf_sc_tianscd23_b200 import xs as X

    rank, world, local = D.env_rank()
    if world != a.gpus:
        raise SystemExit(f"--gpus {a.gpus} but WORLD_SIZE={world}")
    local = local % torch.cuda.device_count()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        if a.backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group("gloo")
    sort = not a.no_sort
    f32 = a.f32
    L_cfg = a.lookups or pre["lookups"]
    # strong scaling of a sorted batch: energy-range shards of all L lookups
    # (each rank keeps the full batch's energy density); otherwise
    # contiguous id ranges (weak: L per rank; strong unsorted: L / R)
    energy_shards = a.scaling == "strong" and sort and world > 1 and a.shard == "energy"
    first, L = (0, L_cfg) if energy_shards else D.shard_range(rank, world, L_cfg, a.scaling)

    t0 = time.time()
    g = X.Grid.from_preset(a.config, device=local)
    torch.cuda.synchronize()
    init_s = time.time() - t0
    stream = torch.cuda.current_stream(dev)

    def lookup(vsum=None, want=()):
        if energy_shards:
            return g.lookup_shard(0, L_cfg, rank, world, want=want, vsum=vsum, f32=f32)
        return g.lookup(first, L, sort=sort, want=want, vsum=vsum, f32=f32)

    # untimed: this rank's lookups (per-material counts for the exact
    # algorithmic work; the inputs of the end-to-end leg)
    vs0, res0 = lookup(want=("mat", "energy"))
    torch.cuda.synchronize()
    if energy_shards:   # positions of other shards are not written: recompute the batch
        _, full = g.lookup(0, L_cfg, want=("mat", "energy"))
        e = full["energy"]
        lo, hi = D.energy_shard_bounds(rank, world)
        sel = (e >= lo) & (e < hi)
        res0 = {"energy": e[sel].contiguous(), "mat": full["mat"][sel].contiguous()}
        del full, e, sel
    n_local = int(vs0[1])
    mats = torch.bincount(res0["mat"].long(), minlength=g.info.n_mats).cpu().tolist()
    num_nucs = g.table(X.XS_TABLE_NUM_NUCS).tolist()
    nuc_lookups = sum(c * n for c, n in zip(mats, num_nucs))
    idx_bytes = 4 if pre["grid_type"] == "unionized" else 8
    gather_bytes = nuc_lookups * (idx_bytes + 96)            # A4 + A5 per launch
    search_probes = math.ceil(math.log2(max(2, g.info.n_union - 1))) \
        if pre["grid_type"] == "unionized" else 0
    search_bytes = n_local * 8 * search_probes
    balg_per_lookup = (gather_bytes + search_bytes) / max(1, n_local)  # SURVEY §8(d) B_alg
    gold = golden().get(a.config)

    vsum = torch.zeros(2, dtype=torch.int64, device=dev)
    a9 = [torch.cuda.Event(enable_timing=True) for _ in range(2 * (a.steps + a.warmup))]
    a9_used = [0]

    def step():
        vsum.zero_()
        lookup(vsum=vsum)
        if world > 1:
            q = a9_used[0]
            if q + 1 < len(a9):
                a9[q].record(stream)
            if a.backend == "nccl":
                D.combine_vsum(vsum)      # A9 over NCCL (NVLink / NVSwitch)
            else:
                vsum.copy_(D.combine_vsum(vsum.cpu()))
            if q + 1 < len(a9):
                a9[q + 1].record(stream)
                a9_used[0] = q + 2

    for _ in range(a.warmup):
        step()
    torch.cuda.synchronize()
    a9_used[0] = 0
    g.timing(True)
    with ClockSampler(local) as clk:
        ms_local, per_step = _timed_steps(step, stream, a.steps, world, dist)
    tm = g.timing_read()
    g.timing(False)
    a9_ms = (sum(a9[q].elapsed_time(a9[q + 1]) for q in range(0, a9_used[0], 2)) /
             max(1, a9_used[0] // 2)) if world > 1 else 0.0
    ms = D.max_over_ranks(ms_local, device=dev if a.backend == "nccl" else None)
    med = statistics.median(per_step)
    med_max = D.max_over_ranks(med, device=dev if a.backend == "nccl" else None)
    total_lookups = L * world * a.steps if a.scaling == "weak" else L_cfg * a.steps
    value = total_lookups / (ms / 1e3)
    vglob = [int(x) for x in vsum.cpu()]
    hash_check = None
    if gold and vglob[1] == gold["lookups"] and (a.scaling == "strong" or world == 1):
        hash_check = vglob == [gold["sum_v_f32" if f32 else "sum_v"], gold["lookups"]]

    peak, peak_src = measured_peaks()
    gather_ms = tm["ms_gather"] / max(1, tm["calls"])
    achieved = gather_bytes / (gather_ms / 1e3) / 1e9
    traffic_per_lookup, traffic_src = ncu_traffic(a.config, sort)
    roofline_hbm = {"bound": "hbm", "kernel": GATHER_KERNEL[sort], "achieved": achieved,
                    "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                    "traffic": traffic_per_lookup * n_local if traffic_per_lookup else None,
                    "peak_source": peak_src,
                    "algorithmic_bytes_per_launch": gather_bytes,
                    "gather_ms_per_launch": gather_ms,
                    "traffic_source": traffic_src,
                    "note": "algorithmic bytes = sum over lookups of n_nuclides(mat) x "
                            f"({idx_bytes} B index + 96 B record pair); on sorted batches the "
                            "pairs are re-read from shared memory and L2, so frac > 1 measures "
                            "reuse, not HBM bandwidth (traffic = DRAM bytes per launch, ncu)"}
    if sort:
        # energy-sorted batches re-read each record pair from shared memory for
        # ~40 lookups: the staged gather is bound by the FP64 pipe
        fp64_peak, fp64_src = fp64_pipe_peak()
        per = FP64_OPS_F32_VARIANT if f32 else FP64_OPS_PER_LOOKUP_NUCLIDE
        ops = nuc_lookups * per
        fp64_achieved = ops / (gather_ms / 1e3) / 1e12
        roofline = {"bound": "alu", "kernel": GATHER_KERNEL[sort], "achieved": fp64_achieved,
                    "peak": fp64_peak, "unit": "TFLOP/s", "frac": fp64_achieved / fp64_peak,
                    "traffic": roofline_hbm["traffic"], "peak_source": fp64_src,
                    "algorithmic_fp64_ops_per_launch": ops,
                    "gather_ms_per_launch": gather_ms, "traffic_source": traffic_src,
                    "note": ("FP64 pipe operations (DADD/DMUL/DFMA count one each): "
                             f"{per} per (lookup, nuclide) = f (1 sub + 3 for the correctly "
                             "rounded division by a precomputed reciprocal) + " +
                             ("1 conversion to binary32; the channels run as binary32 "
                              "FFMA2 (2 per channel pair of lookups)" if f32 else
                              "5 channels x (mul, sub, mul, add)") +
                             "; traffic = DRAM bytes per launch from ncu")}
    else:
        roofline = roofline_hbm
    step_frac = balg_per_lookup * (value / world) / 8e12

    line = {"metric": "XS lookups/sec", "value": value, "unit": "lookups/s", "n_gpus": world,
            "steps": a.steps, "warmup": a.warmup, "ms_per_step": ms / a.steps,
            "ms_per_step_median": med_max,
            "higher_is_better": True, "scaling": a.scaling, "vs_baseline": None,
            "dtype": "f32" if f32 else "f64", "data": "synthetic",
            "config": dict(cfg, shard=("energy ranges [r/R, (r+1)/R) of all L lookups "
                                       "(xs_lookup_batch_shard)" if energy_shards else
                                       "contiguous lookup-id ranges")),
            "roofline": roofline,
            "roofline_hbm": roofline_hbm,
            "hbm_gather_roofline_frac_8TBs": step_frac,
            "balg_bytes_per_lookup": balg_per_lookup,
            "phase_ms_per_step": {k: tm[k] / max(1, tm["calls"])
                                  for k in ("ms_count", "ms_bucket", "ms_gather")},
            "a9_allreduce_ms_per_step": a9_ms,
            "gpu_launches": int(tm["kernel_launches"]),
            "hash": D.global_hash(vglob), "lookups_per_step": vglob[1],
            "oracle_hash": (gold.get("hash_f32" if f32 else "hash") if gold and
                            vglob[1] == gold["lookups"] else None),
            "hash_matches_oracle": hash_check, "init_s": round(init_s, 2),
            "grid_device_bytes": int(g.info.device_bytes)}
    # ------------------------------------------------------------- e2e leg
    if not a.no_e2e:
        # the public call a host program makes: pinned host energy (f64) +
        # material (u8) in, vsum out, every step; XS_FLAG_HOST_ASYNC with two
        # alternating workspaces lets step k's upload overlap step k-1's
        # lookups (the library orders reuse of a workspace)
        e_host = res0["energy"].cpu().pin_memory()
        m_host = res0["mat"].cpu().to(torch.uint8).pin_memory()   # XS_FLAG_MAT_U8
        fl = (X.XS_FLAG_SORT if sort else 0) | X.XS_FLAG_HOST_ASYNC | X.XS_FLAG_MAT_U8
        nws = g.workspace_size(e_host.numel(), fl)
        wss = [torch.empty(nws, dtype=torch.uint8, device=dev)]
        try:  # a second workspace lets consecutive calls overlap (XL: may not fit)
            wss.append(torch.empty(nws, dtype=torch.uint8, device=dev))
        except torch.OutOfMemoryError:
            pass
        vs_h = [torch.zeros(2, dtype=torch.int64).pin_memory() for _ in range(a.e2e_steps + 1)]
        g.lookup_explicit(e_host, m_host, sort=sort, vsum=vs_h[-1], f32=f32, asynchronous=True,
                          workspace=wss[-1])  # warm-up
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        t0 = time.perf_counter()
        for k in range(a.e2e_steps):
            g.lookup_explicit(e_host, m_host, sort=sort, vsum=vs_h[k], f32=f32, asynchronous=True,
                              workspace=wss[k % len(wss)])  # H2D, lookup, D2H of vsum
        torch.cuda.synchronize()
        dt = time.perf_counter() - t0
        dt = D.max_over_ranks(dt, device=dev if a.backend == "nccl" else None)
        e2e_total = L * world * a.e2e_steps if a.scaling == "weak" else L_cfg * a.e2e_steps
        ref = [int(x) for x in vs0]
        line["e2e"] = {"value": e2e_total / dt, "unit": "lookups/s",
                       "h2d_bytes_per_step": int(e_host.numel() * 9), "d2h_bytes_per_step": 16,
                       "api": "xs_lookup_explicit(XS_FLAG_HOST_ASYNC | XS_FLAG_MAT_U8): pinned "
                              "host energy (f64) + material (u8) uploaded and vsum read back "
                              "every step; consecutive steps pipelined over two workspaces; "
                              "wall clock over all steps",
                       "steps": a.e2e_steps, "workspaces": len(wss),
                       "vsum_matches_batch": all([int(x) for x in v] == ref
                                                 for v in vs_h[:a.e2e_steps])}
        del e_host, m_host, wss
    line["clocks"] = clk.summary()
    # ------------------------------------------- single-GPU context legs
    if world == 1 and not a.no_extras:
        if sort and pre["lookups"] >= 1_000_000:
            line["projection_strong"] = {
                "note": "one-GPU projection of strong scaling (L fixed): each rank's shard "
                        "timed alone on this GPU (the lower of two 5-step means), R-GPU "
                        "step = slowest shard; A9 (16-byte all-reduce) not included; weak "
                        "scaling (L per rank, no exchange but A9) projects to R x value",
                **strong_projection(g, L, f32, stream, value, ms / a.steps)}
        # config 3 unsorted and the paper's kernel shape, as context
        if sort and not f32:
            g.timing(True)
            ms_u = _time_fn(lambda: g.lookup(first, L, sort=False), stream, a.extra_steps)
            tmu = g.timing_read()
            g.timing(False)
            gms = tmu["ms_gather"] / max(1, tmu["calls"])
            tr, trs = ncu_traffic(a.config, False)
            ach = gather_bytes / (gms / 1e3) / 1e9
            line["unsorted"] = {
                "value": L / (ms_u / 1e3), "ms_per_step": ms_u, "unit": "lookups/s",
                "roofline": {"bound": "hbm", "kernel": GATHER_KERNEL[False], "achieved": ach,
                             "peak": peak, "unit": "GB/s", "frac": ach / peak,
                             "gather_ms_per_launch": gms,
                             "dram_bytes_per_lookup": tr, "traffic_source": trs,
                             "dram_frac": (tr * L / (gms / 1e3) / 1e9 / peak) if tr else None}}
            ms_b = _time_fn(lambda: g.lookup(first, L, baseline=True), stream, 3, warm=1)
            line["paper_kernel_shape"] = {
                "value": L / (ms_b / 1e3), "ms_per_step": ms_b, "unit": "lookups/s",
                "what": "XS_FLAG_BASELINE: XSBench-CUDA shape (thread per lookup, id order, "
                        "no bucketing), same exact arithmetic, on this B200"}
    if rank == 0 and world == 1 and not a.no_cpu_baseline:
        try:
            rate, cores, desc, S, n = oracle_sample_rate(pre, a.cpu_seconds, f32=f32)
            rate1, _, desc1, _, _ = oracle_sample_rate(pre, a.cpu_seconds / 4, f32=f32, cores=1)
            line["cpu_baseline"] = {"value": rate, "unit": "lookups/s", "cores": cores,
                                    "kind": "oracle", "sample": desc, "cpu": cpu_info(),
                                    "t1_value": rate1, "t1_sample": desc1}
        except Exception as e:  # the oracle is test infrastructure; report, don't fail
            line["cpu_baseline"] = {"value": None, "unit": "lookups/s", "cores": None,
                                    "kind": "oracle", "sample": f"failed: {e}"}
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def _free_port() -> int:
    import socket
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def self_launch(a) -> int | None:
    """`bench.py --gpus N` outside torchrun: start N ranks (one per GPU) with
    torch.distributed.run on 127.0.0.1 and relay rank 0's line."""
    if a.gpus <= 1 or "WORLD_SIZE" in os.environ:
        return None
    import subprocess
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
           f"--nproc-per-node={a.gpus}", "--master-addr", "127.0.0.1",
           "--master-port", str(_free_port()), os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd)


def main():
    a = parse()
    rc = self_launch(a)
    if rc is not None:
        return rc
    if a.config.startswith("rs-"):
        from paper_conf_sc_tianscd23_b200.rs import RS_PRESETS
        pre = dict(RS_PRESETS[a.config])
        per_gpu = a.lookups or pre["lookups"]
        cfg = {"workload": a.config, "app": "RSBench event mode (multipole, doppler)",
               "n_nuclides": pre["n_nuclides"], "avg_n_poles": 1000, "avg_n_windows": 100,
               "lookups_per_gpu": per_gpu if a.scaling == "weak" else None,
               "lookups_total": per_gpu if a.scaling == "strong" else per_gpu * a.gpus,
               "sort": "material + 1024 energy bins" if not a.no_sort else "none",
               "precision": "binary64 (R28)",
               "l2": "not flushed: compute-bound; the 23 MB pole table is L2-resident by design",
               "parallelism": f"dp{a.gpus} (lookup shards, tables replicated)"}
        return run_rs(a, pre, cfg)
    from paper_conf_sc_tianscd23_b200.xs_presets import PRESETS
    pre = dict(PRESETS[a.config])
    per_gpu = a.lookups or pre["lookups"]
    cfg = {"workload": a.config, "n_isotopes": pre["n_isotopes"],
           "n_gridpoints": pre["n_gridpoints"], "grid": pre["grid_type"],
           "hash_bins": pre.get("hash_bins"), "lookups_per_gpu": per_gpu if a.scaling == "weak"
           else None, "lookups_total": per_gpu if a.scaling == "strong" else per_gpu * a.gpus,
           "sort": ("A2 material+energy binning (2^18 energy bins per material)"
                    if not a.no_sort else "none"),
           "precision": ("fp32 variant (R18: binary64 search and weight, binary32 channels "
                         "and accumulation)" if a.f32 else "binary64 (R10, R11)"),
           "l2": "not flushed: the resident tables (GBs, see grid_device_bytes) far exceed "
                 "the 126 MB L2",
           "parallelism": f"dp{a.gpus} (lookup shards, grid replicated)"}
    if a.impl == "reference":
        return run_reference(a, pre, cfg)
    if a.mode == "history":
        return run_history(a, pre, cfg)
    return run_ours(a, pre, cfg)


if __name__ == "__main__":
    sys.exit(main())
