"""GPU parity of history mode (R19):
xs_lookup_history (through the C-ABI) against the oracle's serial particle
chains, element by element — energies, materials, macro XS and v of every
chained lookup bit-exact — and the full XSBench history problem (500,000
particles x 34 lookups) against the oracle's golden sum
(tests/golden/oracle_hashes.json, written by tools/make_golden.py from
oracle/ only)."""
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
WANT = ("macro_xs", "energy", "mat", "verification")

with open(os.path.join(HERE, "golden", "oracle_hashes.json")) as f:
    GOLDEN = json.load(f)


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


def _compare(res, ref):
    out = {k: v.cpu().numpy() for k, v in res.items()}
    assert np.array_equal(out["energy"], ref["p"])
    assert np.array_equal(out["mat"], ref["mat"])
    bad = np.nonzero(~np.all(out["macro_xs"] == ref["M"], axis=1))[0]
    assert bad.size == 0, (bad[:10], out["macro_xs"][bad[:3]], ref["M"][bad[:3]])
    assert np.array_equal(out["verification"], ref["v"])


@pytest.mark.parametrize("sort", [False, True])
@pytest.mark.parametrize("preset", ["tiny", "tiny-hash", "tiny-nuclide"])
def test_tiny_history_full_parity(X, preset, sort):
    grid_type = {"tiny": "unionized", "tiny-hash": "hash", "tiny-nuclide": "nuclide"}[preset]
    g = X.Grid.from_preset("tiny", grid_type=grid_type, hash_bins=128)
    o = _oracle("tiny")
    gold = GOLDEN["tiny"]["history"]
    P, L = gold["particles"], gold["lookups_per_particle"]
    vs, res = g.lookup_history(0, P, L, sort=sort, want=WANT)
    torch.cuda.synchronize()
    S, ref = o.run_history(0, P, L, mode=oracle.UNIONIZED, nthreads=NT, outputs=True)
    assert S == gold["sum_v"]
    assert [int(x) for x in vs.cpu()] == [S, P * L]
    _compare(res, ref)


@pytest.mark.parametrize("P,L,first", [(1, 1, 0), (1, 34, 12345), (33, 7, 3), (1000, 2, 99)])
def test_tiny_history_ragged(X, P, L, first):
    g = X.Grid.from_preset("tiny")
    o = _oracle("tiny")
    vs, res = g.lookup_history(first, P, L, want=WANT)
    torch.cuda.synchronize()
    S, ref = o.run_history(first, P, L, outputs=True)
    assert [int(x) for x in vs.cpu()] == [S, P * L]
    _compare(res, ref)


def test_history_shards_accumulate(X):
    g = X.Grid.from_preset("tiny")
    gold = GOLDEN["tiny"]["history"]
    P, L = gold["particles"], gold["lookups_per_particle"]
    vsum = torch.zeros(2, dtype=torch.int64, device="cuda")
    for a, b in [(0, 1000), (1000, 1001), (1001, 2500), (2500, P)]:
        g.lookup_history(a, b - a, L, vsum=vsum)
    torch.cuda.synchronize()
    assert [int(x) for x in vsum.cpu()] == [gold["sum_v"], P * L]


def test_history_invalid_arguments(X):
    g = X.Grid.from_preset("tiny")
    with pytest.raises(X.XSError):
        g.lookup_history(0, 10, 0)
    with pytest.raises(X.XSError):
        g.lookup_history(0, 10, 3, want=("grid_index",))


@pytest.mark.parametrize("name", ["small", "large", "large-hash"])
def test_full_history_sum_and_samples(X, name):
    gold = GOLDEN[name]["history"]
    P, L = gold["particles"], gold["lookups_per_particle"]
    g = X.Grid.from_preset(name)
    pre = X.PRESETS[name]
    sort = pre.get("sort", False)
    vs, _ = g.lookup_history(0, P, L, sort=sort)
    torch.cuda.synchronize()
    assert [int(x) for x in vs.cpu()] == [gold["sum_v"], P * L]
    # sampled particles, every chained lookup against the oracle
    o = _oracle(name, hash_bins=8192)
    for first, n in [(0, 300), (P // 2, 200), (P - 100, 100)]:
        _, res = g.lookup_history(first, n, L, sort=sort, want=WANT)
        torch.cuda.synchronize()
        S, ref = o.run_history(first, n, L, mode=oracle.HASH, nthreads=NT, outputs=True)
        _compare(res, ref)
