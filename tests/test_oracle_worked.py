"""Oracle pins P6 (hand-worked two-nuclide example), P7 (linear closed form),
P8 (interpolation invariants) and P14 (verification tie cases).

Reference: SURVEY.md §8(c) pins P6-P8, P14; DESIGN.md "Oracle pins".
"""
import json
import os

import numpy as np
import pytest

import oracle

HERE = os.path.dirname(os.path.abspath(__file__))


def _worked():
    with open(os.path.join(HERE, "golden", "worked_two_nuclide.json")) as f:
        return json.load(f)


def _worked_oracle(hash_bins=0):
    w = _worked()
    grid = np.zeros((2, 3, 6))
    for i, name in enumerate(("A", "B")):
        grid[i, :, 0] = w["nuclides"][name]["E"]
        grid[i, :, 1:] = np.array(w["nuclides"][name]["xs"], dtype=np.float64)
    mats = np.array([w["material"]["nuclides"]], np.int32)
    concs = np.array([w["material"]["concs"]], np.float64)
    return w, oracle.Oracle.from_arrays(grid, np.array([2], np.int32), mats, concs,
                                        hash_bins=hash_bins)


def test_worked_union_grid():
    w, o = _worked_oracle()
    assert o.union().tolist() == w["union"]


@pytest.mark.parametrize("case", range(5))
@pytest.mark.parametrize("mode", [oracle.UNIONIZED, oracle.NUCLIDE])
def test_worked_example_exact(case, mode):
    w, o = _worked_oracle()
    c = w["cases"][case]
    p = c["p"]
    for n in range(2):
        assert o.nuclide_bracket(n, p) == c["k"][n]
    M, gi = o.macro_xs(p, 0, mode)
    # dyadic data: bit-exact equality, not a tolerance
    assert M.tolist() == c["M"]
    assert oracle.verify(M) == c["v"]
    if mode == oracle.UNIONIZED:
        assert gi == c["u"]
        assert o.union_index(p) == c["u"]
        if "ig_row" in c:
            assert [o.index_grid_entry(c["u"], n) for n in range(2)] == c["ig_row"]


def test_worked_example_hash_variant():
    w, o = _worked_oracle(hash_bins=4)
    h = w["hash_variant"]
    assert o.hash_bin(h["p"]) == h["b"]
    assert [o.hash_entry(h["b"], n) for n in range(2)] == h["hg_b"]
    assert [o.hash_entry(h["b"] + 1, n) + 1 for n in range(2)] == h["u_hi"]
    assert [o.hash_bracket(h["b"], n, h["p"]) for n in range(2)] == h["k"]
    # hash mode reproduces every worked case bit-exactly as well
    for c in w["cases"]:
        M, b = o.macro_xs(c["p"], 0, oracle.HASH)
        assert M.tolist() == c["M"]


def test_verify_tie_and_negative_cases():
    # P14: equal maxima -> lower channel index wins; all <= -1 -> v = 1
    assert oracle.verify([0.5, 0.5, 0.1, 0.2, 0.3]) == 1
    assert oracle.verify([0.1, 0.7, 0.7, 0.7, 0.2]) == 2
    assert oracle.verify([-2.0, -3.0, -1.5, -1.0, -4.0]) == 1   # -1.0 is not > -1.0
    assert oracle.verify([-2.0, -3.0, -0.5, -1.0, -4.0]) == 3
    assert oracle.verify([0.0, 0.0, 0.0, 0.0, 0.0]) == 1
    assert oracle.verify([1.0, 2.0, 3.0, 4.0, 5.0]) == 5
    assert oracle.verify([-0.0, 0.0, -1e-300, 1e-300, 0.0]) == 4


def _linear_oracle(rng, I=3, N=17):
    """Dyadic linear data: channel c of nuclide n is alpha[n,c]*E + beta[n,c]."""
    # strictly increasing dyadic energies in (0, 1)
    E = np.array([np.sort(rng.choice(np.arange(1, 256), size=N, replace=False)) for _ in range(I)])
    E = E / 256.0
    alpha = rng.integers(-8, 9, size=(I, 5)) / 8.0
    beta = rng.integers(-8, 9, size=(I, 5)) / 4.0
    grid = np.zeros((I, N, 6))
    grid[:, :, 0] = E
    grid[:, :, 1:] = alpha[:, None, :] * E[:, :, None] + beta[:, None, :]
    mats = np.array([list(range(I))], np.int32)
    concs = (rng.integers(1, 16, size=(1, I)) / 16.0)
    return grid, alpha, beta, mats, concs


def test_linear_closed_form():
    # P7: linear channels are reproduced exactly by linear interpolation (and
    # extrapolation), so M_c = sum_j conc_j (alpha_jc p + beta_jc) exactly for
    # dyadic p on a coarse lattice (all products/sums exact in binary64).
    rng = np.random.default_rng(7)
    for _ in range(5):
        grid, alpha, beta, mats, concs = _linear_oracle(rng)
        o = oracle.Oracle.from_arrays(grid, np.array([3], np.int32), mats, concs, hash_bins=8)
        for p in np.arange(0, 257) / 256.0:
            expect = np.zeros(5)
            for j in range(3):
                expect = expect + concs[0, j] * (alpha[j] * p + beta[j])
            for mode in (oracle.UNIONIZED, oracle.NUCLIDE, oracle.HASH):
                M, _ = o.macro_xs(float(p), 0, mode)
                assert np.array_equal(M, expect), (p, mode, M, expect)


def test_interpolation_invariants_tiny():
    # P8 on the tiny config: f in [0,1] for interior p; x_c within the bracket
    # values; p == hi.E reproduces hi exactly; M_c >= 0 when no extrapolation.
    o = oracle.Oracle.from_spec(12, 1000, conc_seed=1070 * 1070, material_rule=1)
    grid = o.grid()
    rng = np.random.default_rng(3)
    for _ in range(3000):
        n = int(rng.integers(0, 12))
        p = float(rng.random())
        k = o.nuclide_bracket(n, p)
        lo, hi = grid[n, k], grid[n, k + 1]
        xs = o.micro_xs(n, k, p)
        if lo[0] <= p <= hi[0]:
            f = (hi[0] - p) / (hi[0] - lo[0])
            assert 0.0 <= f <= 1.0
            for c in range(5):
                a, b = sorted((lo[1 + c], hi[1 + c]))
                assert a - 1e-16 <= xs[c] <= b + 1e-16
    # exact hits: p equal to a grid energy -> bracket starts there (R5) and
    # f == 1, so x = hi - (hi - lo) equals lo up to the rounding of hi - lo
    for n in range(12):
        for k in (0, 1, 500, 998):
            p = float(grid[n, k, 0])
            assert o.nuclide_bracket(n, p) == k
            x = o.micro_xs(n, k, p)
            scale = np.maximum(np.abs(grid[n, k, 1:]), np.abs(grid[n, k + 1, 1:]))
            assert np.all(np.abs(x - grid[n, k, 1:]) <= 2.0**-51 * scale)
        p = float(grid[n, 999, 0])     # last point -> bracket N-2, x = hi exactly
        assert o.nuclide_bracket(n, p) == 998
        assert np.array_equal(o.micro_xs(n, 998, p), grid[n, 999, 1:])
