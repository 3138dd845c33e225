"""GPU parity of the fp32 variant (XS_FLAG_F32, R18) against the
oracle's fp32 variant, element by element, and against the binary64 oracle
within the north_star's fp32 tolerance.

Bars: energy, material, grid index and verification bit-exact; macro XS
bit-exact against the oracle's R18 arithmetic (binary32, one rounding per
operation, blocked accumulation, same order); the verification sum equals
the oracle's fp32 golden sum at full size; against binary64, for EVERY
channel value (north_star "1e-5 if an fp32 variant is offered", in SURVEY
Q12's condition-aware form): |M32 - M64| <= 1e-5 sum_j |x_c conc_j|, and
R18's a-priori bound |M32 - M64| <= (16 + ceil(n/16) + 4) 2^-24 S_c.
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
CONC_SEED = 1070 * 1070
with open(os.path.join(HERE, "golden", "oracle_hashes.json")) as f:
    GOLDEN = json.load(f)
WANT = ("macro_xs", "energy", "mat", "grid_index", "verification")


@pytest.fixture(scope="module")
def X():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_sc_tianscd23_b200.xs as xs
    return xs


def _oracle(name, hash_bins=0):
    g = GOLDEN[name]
    return oracle.Oracle.from_spec(g["n_isotopes"], g["n_gridpoints"], conc_seed=CONC_SEED,
                                   material_rule=g["material_rule"], hash_bins=hash_bins,
                                   nthreads=NT)


@pytest.mark.parametrize("grid_type,bins", [("unionized", 0), ("hash", 97), ("nuclide", 0)])
@pytest.mark.parametrize("sort", [False, True])
def test_tiny_f32_parity(X, grid_type, bins, sort):
    g = X.Grid.from_preset("tiny", grid_type=grid_type, hash_bins=bins)
    mode = {"unionized": oracle.UNIONIZED, "hash": oracle.HASH, "nuclide": oracle.NUCLIDE}[grid_type]
    o = _oracle("tiny", hash_bins=bins)
    S, ref = o.run(0, 100_000, mode=mode | oracle.F32, nthreads=NT, outputs=True)
    vs, res = g.lookup(0, 100_000, sort=sort, want=WANT, f32=True)
    torch.cuda.synchronize()
    out = {k: v.cpu().numpy() for k, v in res.items()}
    assert np.array_equal(out["energy"], ref["p"])
    assert np.array_equal(out["mat"], ref["mat"])
    assert np.array_equal(out["grid_index"], ref["grid_index"])
    bad = np.nonzero(~np.all(out["macro_xs"] == ref["M"], axis=1))[0]
    assert bad.size == 0, (bad[:5], out["macro_xs"][bad[:3]], ref["M"][bad[:3]])
    assert np.array_equal(out["verification"], ref["v"])
    assert [int(x) for x in vs.cpu()] == [S, 100_000]
    assert S == GOLDEN["tiny"]["sum_v_f32"]
    # the north_star tolerance against binary64, element-wise
    _check_vs_binary64(o, 0, 100_000, mode, out["macro_xs"], ref["mat"])


def _check_vs_binary64(o, first, count, mode, M32, mat):
    """Element-wise: Q12's 1e-5 and R18's a-priori bound against binary64."""
    _, r64 = o.run(first, count, mode=mode, nthreads=NT, outputs=True)
    _, ra = o.run(first, count, mode=oracle.SCALE_A, nthreads=NT, outputs=True)
    _, rs = o.run(first, count, mode=oracle.SCALE_S, nthreads=NT, outputs=True)
    d = np.abs(M32 - r64["M"])
    q12 = d / ra["M"]
    assert q12.max() <= 1e-5, (q12.max(), np.unravel_index(q12.argmax(), q12.shape))
    n = o.num_nucs()[mat].astype(np.float64)
    factor = (16 + np.ceil(n / 16) + 4) * 2.0 ** -24
    assert np.all(d <= factor[:, None] * rs["M"])
    return q12.max()


@pytest.mark.parametrize("variant", [0, 31, 32, 33, 34, 36, 46, 47, 48])
@pytest.mark.parametrize("first,count", [(0, 1), (5, 31), (999_999, 4097), (3, 70_001)])
def test_f32_shapes_and_ragged(X, variant, first, count):
    g = X.Grid.from_preset("tiny")
    g.set_param("variant", variant)
    S, ref = _oracle("tiny").run(first, count, mode=oracle.UNIONIZED | oracle.F32, nthreads=NT,
                                 outputs=True)
    vs, res = g.lookup(first, count, sort=True, want=("macro_xs", "verification"), f32=True)
    torch.cuda.synchronize()
    assert np.array_equal(res["macro_xs"].cpu().numpy(), ref["M"])
    assert np.array_equal(res["verification"].cpu().numpy(), ref["v"])
    assert [int(x) for x in vs.cpu()] == [S, count]


def test_f32_explicit_host_io(X):
    g = X.Grid.from_preset("tiny")
    o = _oracle("tiny")
    rng = np.random.default_rng(9)
    p = rng.random(20_000)
    p[:4] = [0.0, 1.0, -0.25, 1.5]      # both grid ends, extrapolation
    m = rng.integers(0, 12, 20_000).astype(np.int32)
    S, M, v = o.run_explicit(p, m, mode=oracle.UNIONIZED | oracle.F32, nthreads=NT)
    vs, res = g.lookup_explicit(torch.tensor(p), torch.tensor(m), sort=True,
                                want=("macro_xs", "verification"), f32=True)
    assert np.array_equal(res["macro_xs"].numpy(), M)
    assert np.array_equal(res["verification"].numpy(), v)
    assert [int(x) for x in vs] == [S, 20_000]


@pytest.mark.parametrize("name", ["small", "large", "large-hash"])
def test_full_config_f32_hash(X, name):
    gold = GOLDEN[name]
    g = X.Grid.from_preset(name)
    L = gold["lookups"]
    vs, res = g.lookup(0, L, sort=True, want=("energy", "mat"), f32=True)
    torch.cuda.synchronize()
    assert [int(x) for x in vs.cpu()] == [gold["sum_v_f32"], L]
    rng = np.random.default_rng(1)
    ids = np.unique(np.concatenate([[0, L - 1], rng.integers(0, L, 1500)]))
    ids_t = torch.tensor(ids, device="cuda")
    E = res["energy"][ids_t].cpu().numpy()
    mt = res["mat"][ids_t].cpu().numpy()
    _, rex = g.lookup_explicit(torch.tensor(E, device="cuda"), torch.tensor(mt, device="cuda"),
                               want=("macro_xs",), f32=True)
    Mx = rex["macro_xs"].cpu().numpy()
    o = _oracle(name, hash_bins=X.PRESETS[name].get("hash_bins", 0))
    mode = oracle.HASH if X.PRESETS[name]["grid_type"] == "hash" else oracle.UNIONIZED
    _, M, _ = o.run_explicit(E, mt, mode=mode | oracle.F32, nthreads=NT)
    assert np.array_equal(Mx, M)


@pytest.mark.parametrize("name", ["large"])
def test_full_config_f32_every_lookup(X, name):
    """All 17M lookups of the sorted fp32 batch (bench --f32's launch):
    bit-exact against the oracle's R18 and within the north_star's 1e-5
    (Q12, element-wise) of binary64 — fuel has 321 nuclides here."""
    gold = GOLDEN[name]
    L = gold["lookups"]
    g = X.Grid.from_preset(name)
    vs, res = g.lookup(0, L, sort=True, want=("macro_xs", "verification"), f32=True)
    torch.cuda.synchronize()
    M32 = res["macro_xs"].cpu().numpy()
    v32 = res["verification"].cpu().numpy()
    del res
    g.close()
    assert [int(x) for x in vs.cpu()] == [gold["sum_v_f32"], L]
    o = _oracle(name, hash_bins=8192)
    S, ref = o.run(0, L, mode=oracle.HASH | oracle.F32, nthreads=NT, outputs=True)
    bad = np.nonzero(~np.all(M32 == ref["M"], axis=1))[0]
    assert bad.size == 0, (bad[:5], M32[bad[:3]], ref["M"][bad[:3]])
    assert np.array_equal(v32, ref["v"])
    worst = _check_vs_binary64(o, 0, L, oracle.HASH, M32, ref["mat"])
    assert worst < 1e-5


def test_f32_rejects_baseline(X):
    g = X.Grid.from_preset("tiny")
    with pytest.raises(X.XSError) as e:
        g.lookup(0, 100, baseline=True, f32=True)
    assert e.value.status == 4
