"""GPU parity of the RSBench path (include/rs.h, csrc/rs_lookup.cu) against the
CPU oracle (oracle/rs_oracle.c), element by element on the same seeded inputs
(R20-R28).

Bars:
  * energy, material, verification v and the verification sum/hash:
    bit-exact (the argmax is taken on values that agree to ~1e-13);
  * macro XS: |M_gpu - M_oracle| <= RTOL * (1 + |M_oracle|) with
    RTOL = 1e-11 (R28-R30: the kernels keep the oracle's
    operation order up to FMA contraction and ~1-ulp divisions, evaluate
    e^{12iZ} and the phase factors in algebraically equal forms, and use
    CUDA's sin/cos — a few ulp, amplified near the removable singularities
    of the Abrarov series; observed max 1e-13).
"""
import json
import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import oracle  # noqa: E402

HERE = os.path.dirname(os.path.abspath(__file__))
NT = max(1, min(16, os.cpu_count() or 1))
RTOL = 1e-11

with open(os.path.join(HERE, "golden", "rs_oracle_sums.json")) as f:
    GOLDEN = json.load(f)


@pytest.fixture(scope="module")
def R():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_sc_tianscd23_b200.rs as rs
    return rs


_ORACLES = {}
_PROBLEMS = {}


def oracle_for(name):
    if name not in _ORACLES:
        g = GOLDEN[name]
        _ORACLES[name] = oracle.RSOracle(g["n_nuclides"], 1000, 100, 4, g["material_rule"], 42,
                                         1070, g["doppler"])
    return _ORACLES[name]


def problem_for(R, name):
    if name not in _PROBLEMS:
        g = GOLDEN[name]
        _PROBLEMS[name] = R.RSProblem.from_spec(n_nuclides=g["n_nuclides"],
                                                material_rule=g["material_rule"],
                                                doppler=g["doppler"])
    return _PROBLEMS[name]


def _run(p, first, count, **kw):
    vsum, res = p.lookup(first, count, want=("macro_xs", "mat", "energy"), **kw)
    torch.cuda.synchronize()
    return [int(x) for x in vsum.cpu()], {k: v.cpu().numpy() for k, v in res.items()}


def _check_close(M, ref):
    err = np.abs(M - ref) / (1.0 + np.abs(ref))
    assert np.isfinite(M).all()
    assert err.max() <= RTOL, f"max scaled error {err.max():.3e}"
    return err.max()


@pytest.mark.parametrize("mode", ["sort", "idorder", "baseline"])
def test_rs_tiny_full(R, mode):
    o = oracle_for("rs-tiny")
    p = problem_for(R, "rs-tiny")
    L = GOLDEN["rs-tiny"]["lookups"]
    S, ref = o.run(0, L, nthreads=NT, outputs=True)
    assert S == GOLDEN["rs-tiny"]["sum_v"]
    kw = dict(sort=mode == "sort", baseline=mode == "baseline")
    vs, out = _run(p, 0, L, **kw)
    assert vs == [S, L]
    assert np.array_equal(out["energy"], ref["E"])
    assert np.array_equal(out["mat"], ref["mat"])
    _check_close(out["macro_xs"], ref["M"])
    v = np.argmax(out["macro_xs"], axis=1) + 1     # first maximum, as R27
    assert np.array_equal(v, ref["v"])


def test_rs_tiny_nodoppler(R):
    o = oracle_for("rs-tiny-nodoppler")
    p = problem_for(R, "rs-tiny-nodoppler")
    L = 20_000
    S, ref = o.run(0, L, nthreads=NT, outputs=True)
    vs, out = _run(p, 0, L, sort=True)
    assert vs == [S, L]
    _check_close(out["macro_xs"], ref["M"])
    vs, _ = _run(p, 0, GOLDEN["rs-tiny-nodoppler"]["lookups"], sort=True)
    assert vs[0] == GOLDEN["rs-tiny-nodoppler"]["sum_v"]


def test_rs_sorted_equals_idorder_bitwise(R):
    p = problem_for(R, "rs-tiny")
    vs1, a = _run(p, 5, 77_777, sort=True)
    vs2, b = _run(p, 5, 77_777, sort=False)
    assert vs1 == vs2
    for k in a:
        assert np.array_equal(a[k], b[k]), k


def test_rs_shards_and_ragged(R):
    p = problem_for(R, "rs-tiny")
    S = GOLDEN["rs-tiny"]["sum_v"]
    total = 0
    for first, n in ((0, 1), (1, 255), (256, 33_333), (33_589, 66_411)):
        vs, _ = _run(p, first, n, sort=True)
        assert vs[1] == n
        total += vs[0]
    assert total == S
    vs, _ = p.lookup(0, 0)                                # count 0: no-op
    torch.cuda.synchronize()
    assert [int(x) for x in vs.cpu()] == [0, 0]


def test_rs_large_ids(R):
    o = oracle_for("rs-tiny")
    p = problem_for(R, "rs-tiny")
    first = (1 << 40) + 12345
    S, ref = o.run(first, 3000, nthreads=NT, outputs=True)
    vs, out = _run(p, first, 3000, sort=True)
    assert vs == [S, 3000]
    _check_close(out["macro_xs"], ref["M"])


@pytest.mark.parametrize("name", ["rs-small", "rs-large"])
def test_rs_full_workload_sum(R, name):
    """The bench configuration (10M lookups, sorted) against the oracle's
    golden verification sum, plus sampled lookups element by element."""
    g = GOLDEN[name]
    p = problem_for(R, name)
    L = g["lookups"]
    vs, _ = p.lookup(0, L, sort=True)
    torch.cuda.synchronize()
    vs = [int(x) for x in vs.cpu()]
    assert vs == [g["sum_v"], L]
    for key, S in g["shard_sums"].items():
        f, n = (int(x) for x in key.split("+"))
        v2, out = _run(p, f, n, sort=True)
        assert v2 == [S, n]
    o = oracle_for(name)
    rng = np.random.default_rng(0)
    ids = np.sort(rng.choice(L, 400, replace=False))
    _, out = _run(p, 0, L, sort=True)
    for i in ids:
        r = o.lookup(int(i))
        assert out["energy"][i] == r["E"] and out["mat"][i] == r["mat"]
        err = np.abs(out["macro_xs"][i] - r["M"]) / (1.0 + np.abs(r["M"]))
        assert err.max() <= RTOL, (i, err)


def test_rs_workspace_errors(R):
    import paper_conf_sc_tianscd23_b200.xs as X
    p = problem_for(R, "rs-tiny")
    vsum = torch.zeros(2, dtype=torch.int64, device="cuda")
    o = R.rs_outputs(None, None, None, vsum.data_ptr())
    st = torch.cuda.current_stream().cuda_stream
    with pytest.raises(X.XSError) as e:
        R.rs_lookup_batch(p._h, 0, 1000, R.RS_FLAG_SORT, o, None, 0, st)
    assert e.value.status == 1
    with pytest.raises(X.XSError):
        R.rs_lookup_batch(p._h, 0, 1000, 0x80, o, None, 0, st)


def test_rs_bench_multirank_path_on_one_gpu(R):
    """bench.py --config rs-tiny on two ranks sharing the GPU over gloo: shards,
    barrier, max-over-ranks and the vsum all-reduce; the global sum equals
    the oracle's over both shards (weak scaling: ids [0, 2L))."""
    import subprocess
    import sys
    root = os.path.dirname(HERE)
    L = GOLDEN["rs-tiny"]["lookups"]
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
                        "--nproc-per-node", "2", "--master-addr", "127.0.0.1", "--master-port",
                        "29543", "bench.py", "--gpus", "2", "--backend", "gloo", "--config",
                        "rs-tiny", "--scaling", "weak", "--steps", "3", "--warmup", "3",
                            "--no-cpu-baseline"],
                       cwd=root, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["lookups_per_step"] == 2 * L
    S = oracle_for("rs-tiny").run(0, 2 * L, nthreads=NT)
    assert d["hash"] == S % 999983


@pytest.mark.parametrize("sort", [True, False])
def test_rs_explicit_equals_sampled(R, sort):
    """rs_lookup_explicit on the (energy, material) pairs of a sampled batch
    gives the sampled batch's results bit for bit; device and host buffers."""
    p = problem_for(R, "rs-tiny")
    L = 30_000
    vs0, ref = _run(p, 0, L, sort=True)
    e = torch.tensor(ref["energy"], device="cuda")
    m = torch.tensor(ref["mat"].astype(np.uint8), device="cuda")
    vs, res = p.lookup_explicit(e, m, sort=sort, want=("macro_xs", "mat", "energy"))
    torch.cuda.synchronize()
    assert [int(x) for x in vs.cpu()] == vs0
    assert np.array_equal(res["macro_xs"].cpu().numpy(), ref["macro_xs"])
    assert np.array_equal(res["mat"].cpu().numpy(), ref["mat"])
    vh, rh = p.lookup_explicit(e.cpu().pin_memory(), m.cpu().pin_memory(), sort=sort,
                               want=("macro_xs",))
    assert [int(x) for x in vh] == vs0
    assert np.array_equal(rh["macro_xs"].numpy(), ref["macro_xs"])


def test_rs_explicit_invalid_and_oracle(R):
    """Random explicit pairs against the oracle's macro XS; lookups outside the
    domain (mat >= 12, E outside [0, 1], NaN) are skipped with NaN outputs."""
    o = oracle_for("rs-tiny")
    p = problem_for(R, "rs-tiny")
    rng = np.random.default_rng(3)
    E = rng.random(5000)
    E[:4] = [0.0, 1.0, 0.5, np.nextafter(1.0, 0.0)]
    M = rng.integers(0, 12, E.size).astype(np.uint8)
    bad = np.zeros(E.size, bool)
    for i, (e, m) in enumerate([(-0.1, 3), (1.5, 3), (np.nan, 0), (0.3, 12), (0.3, 255)]):
        E[10 + i], M[10 + i] = e, m
        bad[10 + i] = True
    for sort in (True, False):
        vs, res = p.lookup_explicit(torch.tensor(E, device="cuda"), torch.tensor(M, device="cuda"),
                                    sort=sort, want=("macro_xs",))
        torch.cuda.synchronize()
        X = res["macro_xs"].cpu().numpy()
        assert np.isnan(X[bad]).all()
        ref = np.array([o.macro_xs(float(E[i]), int(M[i])) for i in np.flatnonzero(~bad)])
        _check_close(X[~bad], ref)
        v = np.argmax(ref, axis=1) + 1
        assert [int(x) for x in vs.cpu()] == [int(v.sum()), int((~bad).sum())]


def test_rs_sparse_poles_config(R):
    """More windows than poles (empty windows, end < start) and a non-default
    pole count: GPU equals the oracle."""
    o = oracle.RSOracle(12, 5, 50, 4, 1, 42, 1070, 1)
    p = R.RSProblem.from_spec(n_nuclides=12, avg_n_poles=5, avg_n_windows=50, material_rule=1)
    L = 20_000
    S, ref = o.run(0, L, nthreads=NT, outputs=True)
    for sort in (True, False):
        vs, out = _run(p, 0, L, sort=sort)
        assert vs == [S, L]
        _check_close(out["macro_xs"], ref["M"])
    n_nuc, n_pole = p.work_count(0, L)
    assert n_nuc == int(sum(o.num_nucs()[m] for m in ref["mat"]))
    p.close()
