"""Oracle pins for sampling and search: P1 (fast-forward = n-fold stepping),
P3 (pick_mat thresholds and material frequencies), P4 (search = brute-force
linear scan), P5 (XSBench incremental index-grid sweep = definition), P9
(UNIONIZED == NUCLIDE == HASH), plus the hash edge cases R7/R8.

Reference: SURVEY.md §8(c) C2-C3, pins P1, P3-P5, P9; R2-R9.
"""
import math

import numpy as np
import pytest

import oracle

M63 = 1 << 63
A, Cc = 2806196910506780709, 1


def test_lcg_step_closed_form():
    # the step is an affine map mod 2^63, checked with exact Python integers
    for s in (0, 1, 42, 1070, M63 - 1, 123456789123456789):
        assert oracle.lcg_step(s) == (A * s + Cc) % M63
    assert oracle.lcg_to_double(1 << 62) == 0.5
    assert oracle.lcg_to_double(0) == 0.0
    # round-to-nearest conversion: the top 2^9 - 1 states map to exactly 1.0
    assert oracle.lcg_to_double(M63 - 1) == 1.0
    assert oracle.lcg_to_double(M63 - 1024) < 1.0


def test_fast_forward_equals_stepping():
    # P1: FF(s, n) = LCG^n(s) (brute force) and FF(s, a + b) = FF(FF(s, a), b)
    for s in (0, 1, 1070, 42, M63 - 5):
        x = s
        for n in range(2000):
            assert oracle.fast_forward(s, n) == x
            x = oracle.lcg_step(x)
    rng = np.random.default_rng(0)
    for _ in range(200):
        s = int(rng.integers(0, 2**62))
        a = int(rng.integers(0, 2**40))
        b = int(rng.integers(0, 2**40))
        assert oracle.fast_forward(s, a + b) == oracle.fast_forward(oracle.fast_forward(s, a), b)
    # a closed form for the affine power: LCG^n(s) = a^n s + c (a^n - 1)/(a - 1)
    for n in (1, 2, 3, 1000, 2**20 + 7, 2 * 16_999_999):
        an = pow(A, n, M63 * (A - 1))
        geo = (an - 1) // (A - 1)
        for s in (1070, 7):
            assert oracle.fast_forward(s, n) == (pow(A, n, M63) * s + geo * Cc) % M63


def test_sample_first_lookups_by_stepping():
    # lookup i uses draws 2i+1 and 2i+2 of the stream from the lookup seed
    x = 1070
    for i in range(300):
        x1 = oracle.lcg_step(x)
        x2 = oracle.lcg_step(x1)
        p, m = oracle.sample(1070, i)
        assert p == x1 / 2.0**63
        assert m == oracle.pick_mat(x2 / 2.0**63)
        x = x2


THRESH_HEX = {  # SURVEY.md Appendix A (reverse-order running sums as binary64)
    1: "0x1.a9fbe76c8b439p-5", 2: "0x1.4ed916872b021p-2", 3: "0x1.d810624dd2f1bp-2",
    4: "0x1.3ae147ae147afp-1", 5: "0x1.5ba5e353f7ceep-1", 6: "0x1.7d70a3d70a3d8p-1",
    7: "0x1.999999999999ap-1", 8: "0x1.9db22d0e56042p-1", 9: "0x1.a5604189374bdp-1",
    10: "0x1.b22d0e560418ap-1", 11: "0x1.b8d4fdf3b645bp-1"}


def test_thresholds_hex():
    T = oracle.thresholds()
    assert T[0] == 0.0
    for m, h in THRESH_HEX.items():
        assert T[m] == float.fromhex(h), m
    # ... and they are the decimal cumulative fractions to within rounding
    dec = np.cumsum([0, .052, .275, .134, .154, .064, .066, .055, .008, .015, .025, .013])
    assert np.allclose(T, dec, rtol=0, atol=1e-15)


def test_pick_mat_boundaries():
    T = oracle.thresholds()
    assert oracle.pick_mat(0.0) == 1
    for m in range(1, 12):
        assert oracle.pick_mat(np.nextafter(T[m], 0)) == m
        assert oracle.pick_mat(T[m]) == (m + 1 if m < 11 else 0)
    assert oracle.pick_mat(0.999) == 0
    assert oracle.pick_mat(1.0) == 0


def test_material_frequencies():
    # P3: frequencies of 2e5 sampled lookups within 5 sigma of the pick
    # distribution (fuel gets 1 - 0.861 = 0.139)
    o = oracle.Oracle.from_spec(12, 2, conc_seed=1, material_rule=1)
    n = 200_000
    _, out = o.run(0, n, mode=oracle.NUCLIDE, nthreads=4, outputs=True)
    freq = np.bincount(out["mat"], minlength=12) / n
    prob = np.array([0.139, .052, .275, .134, .154, .064, .066, .055, .008, .015, .025, .013])
    sigma = np.sqrt(prob * (1 - prob) / n)
    assert np.all(np.abs(freq - prob) < 5 * sigma), (freq, prob)
    # energies uniform in [0, 1): mean and variance within 5 sigma
    p = out["p"]
    assert abs(p.mean() - 0.5) < 5 * math.sqrt(1 / 12 / n)
    assert p.min() >= 0.0 and p.max() < 1.0


def _micro_grid(rng, I, N, integer_energies=False):
    if integer_energies:
        E = np.array([np.sort(rng.choice(np.arange(1, 64), size=N, replace=False))
                      for _ in range(I)]) / 64.0
    else:
        E = np.sort(rng.random((I, N)), axis=1)
    grid = np.zeros((I, N, 6))
    grid[:, :, 0] = E
    grid[:, :, 1:] = rng.random((I, N, 5))
    nmat = 3
    mx = I
    mats = np.full((nmat, mx), -1, np.int32)
    num = np.zeros(nmat, np.int32)
    for m in range(nmat):
        k = int(rng.integers(1, I + 1))
        ids = rng.permutation(I)[:k]
        mats[m, :k] = ids
        num[m] = k
    concs = np.where(mats >= 0, rng.random((nmat, mx)), 0.0)
    return grid, num, mats, concs


def _probes(grid, U, B):
    E = grid[:, :, 0].ravel()
    edges = np.arange(B + 1) / B if B else np.array([])
    base = [0.0, 1.0, np.nextafter(1.0, 0), 1e-300, -0.0]
    return np.concatenate([base, E, np.nextafter(E, 0), np.nextafter(E, 2), edges,
                           np.nextafter(edges, 0), U[:1] / 2, [U[-1] + 1e-3]])


@pytest.mark.parametrize("seed", range(6))
def test_search_brute_force(seed):
    # P4: every search equals a linear scan #{x <= p} - 1, clamped
    rng = np.random.default_rng(seed)
    I, N = int(rng.integers(1, 9)), int(rng.integers(2, 40))
    B = int(rng.integers(1, 50))
    grid, num, mats, concs = _micro_grid(rng, I, N, integer_energies=seed % 2 == 0)
    o = oracle.Oracle.from_arrays(grid, num, mats, concs, hash_bins=B)
    U = o.union()
    assert np.array_equal(U, np.sort(grid[:, :, 0].ravel()))
    for p in _probes(grid, U, B):
        p = float(p)
        u_bf = min(max(int(np.sum(U <= p)) - 1, 0), len(U) - 2)
        assert o.union_index(p) == u_bf
        b = o.hash_bin(p)
        assert b == min(int(p / (1.0 / B)), B - 1)
        for n in range(I):
            k_bf = min(max(int(np.sum(grid[n, :, 0] <= p)) - 1, 0), N - 2)
            assert o.nuclide_bracket(n, p) == k_bf
            assert o.index_grid_entry(u_bf, n) == k_bf            # unionized route
            if p >= 0:
                assert o.hash_bracket(b, n, p) == k_bf            # hash route
    for b in range(B):
        for n in range(I):
            e = b * (1.0 / B)
            assert o.hash_entry(b, n) == min(max(int(np.sum(grid[n, :, 0] <= e)) - 1, 0), N - 2)


def test_grid_search_shape():
    A = np.array([0.1, 0.2, 0.2, 0.3, 0.5])
    for q in (0.0, 0.1, 0.15, 0.2, 0.25, 0.3, 0.4, 0.5, 0.9):
        lo = oracle.grid_search(A, 0, len(A) - 1, q)
        assert lo == min(max(int(np.sum(A <= q)) - 1, 0), len(A) - 2)
        assert oracle.upper_bound(A, q) == int(np.sum(A <= q))


@pytest.mark.parametrize("seed", range(4))
def test_index_grid_sweep_equals_definition(seed):
    # P5: XSBench's incremental construction = clamp(ub(E_n, U[e]) - 1)
    rng = np.random.default_rng(100 + seed)
    I, N = int(rng.integers(1, 7)), int(rng.integers(2, 30))
    grid, num, mats, concs = _micro_grid(rng, I, N, integer_energies=seed % 2 == 0)
    o = oracle.Oracle.from_arrays(grid, num, mats, concs)
    IG = o.index_grid_sweep()
    for e in range(o.NU):
        for n in range(I):
            assert IG[e, n] == o.index_grid_entry(e, n)


def test_index_grid_sweep_tiny_config():
    o = oracle.Oracle.from_spec(12, 1000, conc_seed=1070 * 1070, material_rule=1)
    IG = o.index_grid_sweep()
    rng = np.random.default_rng(1)
    for e in rng.integers(0, o.NU, 4000):
        for n in range(12):
            assert IG[e, n] == o.index_grid_entry(int(e), n)
    for e in (0, 1, o.NU - 2, o.NU - 1):
        for n in range(12):
            assert IG[e, n] == o.index_grid_entry(e, n)


def test_hash_quirk_reading():
    # R7: p equal to a grid energy that lies exactly on a bin edge with
    # u_lo > 0.  XSBench would return bracket 0; the definition (and this
    # oracle) returns u_lo.
    grid = np.zeros((1, 4, 6))
    grid[0, :, 0] = [0.125, 0.25, 0.5, 0.75]
    grid[0, :, 1:] = np.arange(20).reshape(4, 5)
    o = oracle.Oracle.from_arrays(grid, np.array([1], np.int32), np.array([[0]], np.int32),
                                  np.array([[1.0]]), hash_bins=4)
    b = o.hash_bin(0.5)
    assert b == 2 and o.hash_entry(2, 0) == 2
    assert o.hash_bracket(2, 0, 0.5) == 2 == o.nuclide_bracket(0, 0.5)
    # p = 1.0 (R8): bin clamped to B-1, bracket N-2
    assert o.hash_bin(1.0) == 3
    assert o.hash_bracket(3, 0, 1.0) == 2 == o.nuclide_bracket(0, 1.0)


def test_modes_agree_tiny_config():
    # P9: the three routes give bit-identical M (and hence v) on the tiny config
    o = oracle.Oracle.from_spec(12, 1000, conc_seed=1070 * 1070, material_rule=1, hash_bins=97)
    Su, ou = o.run(0, 20000, mode=oracle.UNIONIZED, nthreads=4, outputs=True)
    Sn, on = o.run(0, 20000, mode=oracle.NUCLIDE, nthreads=4, outputs=True)
    Sh, oh = o.run(0, 20000, mode=oracle.HASH, nthreads=4, outputs=True)
    assert Su == Sn == Sh
    assert np.array_equal(ou["M"], on["M"]) and np.array_equal(ou["M"], oh["M"])
    assert np.array_equal(ou["v"], oh["v"])
    assert np.all(oh["grid_index"] == np.minimum((oh["p"] / (1.0 / 97)).astype(np.int64), 96))
