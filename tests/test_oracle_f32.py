"""Pins of the oracle's fp32 variant (R18; north_star "1e-5 if an
fp32 variant is offered").

R18 keeps the binary64 search and interpolation weight and runs the channel
arithmetic, the concentrations and the accumulation in binary32, one
rounding per operation (x = fma(-f, d, hi); block sums B = fma(x, conc, B)
over 16 consecutive nuclides, added to M after each block).  Pins that
do not re-type the formula:
  * the hand-worked two-nuclide example (dyadic with few
    significant bits, so every value is exact in binary32 as well): the fp32
    variant must reproduce the binary64 expected values bit for bit, in all
    three search routes (interior, both extrapolations, exact grid hits);
  * the linear closed form (P7) on dyadic data exact in binary32;
  * an a-priori rounding-error bound against the binary64 oracle on the tiny
    and (sampled) large configs: |M32 - M64| <= (K + ceil(n/K) + 4) 2^-24
    sum_j s_j with K = 16 and s_j = conc_j (|hi.c| + |f| (|hi.c| + |lo.c|))
    (R18) — a dropped term, a wrong sign or index, an unblocked
    accumulation or one in the wrong precision breaks it — and that bound is
    below the north_star's 1e-5 for every material;
  * the north_star's 1e-5 element-wise in SURVEY Q12's condition-aware form,
    |M32 - M64| <= 1e-5 sum_j |x_c conc_j|, on every tiny lookup;
  * every result is a binary32 value (the accumulation really is binary32),
    and the tiny config's verification values agree with binary64 except at
    near-ties.
"""
import numpy as np
import pytest

import oracle
from test_oracle_worked import _linear_oracle, _worked_oracle

U32 = 2.0 ** -24
K = 16   # R18's accumulation block


def bound_factor(n: int) -> float:
    """R18's a-priori error factor for an n-nuclide material (R18)."""
    return (K + -(-n // K) + 4) * U32


@pytest.mark.parametrize("mode", [oracle.UNIONIZED, oracle.NUCLIDE, oracle.HASH])
def test_worked_example_f32_exact(mode):
    w, o = _worked_oracle(hash_bins=4)
    for c in w["cases"]:
        M, gi = o.macro_xs(c["p"], 0, mode | oracle.F32)
        assert M.tolist() == c["M"], (c["p"], M)
        assert oracle.verify(M) == c["v"]


def test_linear_closed_form_f32():
    rng = np.random.default_rng(11)
    for _ in range(4):
        grid, alpha, beta, mats, concs = _linear_oracle(rng)
        o = oracle.Oracle.from_arrays(grid, np.array([3], np.int32), mats, concs, hash_bins=8)
        for p in np.arange(0, 257) / 256.0:
            expect = np.zeros(5)
            for j in range(3):
                expect = expect + concs[0, j] * (alpha[j] * p + beta[j])
            for mode in (oracle.UNIONIZED, oracle.NUCLIDE, oracle.HASH):
                M, _ = o.macro_xs(float(p), 0, mode | oracle.F32)
                assert np.array_equal(M, expect), (p, mode, M, expect)


def _bound_check(o, ids):
    grid, mats, concs, nn = o.grid(), o.mats(), o.concs(), o.num_nucs()
    worst = 0.0
    for i in ids:
        r64 = o.lookup(int(i), oracle.UNIONIZED)
        r32 = o.lookup(int(i), oracle.UNIONIZED | oracle.F32)
        assert (r32["p"], r32["mat"], r32["grid_index"]) == (r64["p"], r64["mat"],
                                                             r64["grid_index"])
        M32 = r32["M"]
        assert np.array_equal(M32.astype(np.float32).astype(np.float64), M32)
        p, m = r64["p"], r64["mat"]
        scale = np.zeros(5)
        for j in range(nn[m]):
            n = mats[m, j]
            k = o.nuclide_bracket(n, p)
            lo, hi = grid[n, k], grid[n, k + 1]
            f = (hi[0] - p) / (hi[0] - lo[0])
            scale += concs[m, j] * (np.abs(hi[1:]) + abs(f) * (np.abs(hi[1:]) + np.abs(lo[1:])))
        A, S = o.macro_scales(p, m)
        assert np.allclose(S, scale, rtol=1e-12, atol=0)   # the oracle's scale = this one
        ratio = np.max(np.abs(M32 - r64["M"]) / (bound_factor(nn[m]) * scale))
        assert ratio <= 1.0, (i, M32, r64["M"])
        worst = max(worst, ratio)
    return worst


def test_f32_bound_below_north_star():
    """The a-priori factor is below 1e-5 for every material of every config
    (fuel: 321 nuclides in large/XL)."""
    for I, rule in ((12, 1), (68, 0), (355, 0)):
        for n in oracle.gen_num_nucs(I, rule):
            assert bound_factor(int(n)) <= 1e-5, (I, n)
    assert bound_factor(321) < 2.5e-6


def test_f32_error_bound_tiny():
    o = oracle.Oracle.from_spec(12, 1000, conc_seed=1070 * 1070, material_rule=1)
    worst = _bound_check(o, range(0, 100_000, 37))
    assert worst > 0.0  # the variant really rounds (it is not the binary64 path)


def test_f32_error_bound_large_sampled():
    o = oracle.Oracle.from_spec(355, 11303, conc_seed=1070 * 1070, material_rule=0)
    rng = np.random.default_rng(5)
    _bound_check(o, rng.integers(0, 17_000_000, 150))


def test_f32_tiny_run_consistent():
    o = oracle.Oracle.from_spec(12, 1000, conc_seed=1070 * 1070, material_rule=1)
    S64, r64 = o.run(0, 100_000, mode=oracle.UNIONIZED, nthreads=4, outputs=True)
    S32, r32 = o.run(0, 100_000, mode=oracle.UNIONIZED | oracle.F32, nthreads=4, outputs=True)
    Sh, rh = o.run(0, 100_000, mode=oracle.NUCLIDE | oracle.F32, nthreads=4, outputs=True)
    assert np.array_equal(r32["M"], rh["M"]) and S32 == Sh   # route-independent (P9)
    # verification differs from binary64 only where two channels nearly tie
    diff = np.nonzero(r32["v"] != r64["v"])[0]
    for i in diff:
        M = np.sort(r64["M"][i])[::-1]
        assert M[0] - M[1] <= 1e-5 * abs(M[0])
    # the north_star's fp32 tolerance, element-wise, condition-aware (Q12)
    _, ra = o.run(0, 100_000, mode=oracle.SCALE_A, nthreads=4, outputs=True)
    q12 = np.abs(r32["M"] - r64["M"]) / ra["M"]
    assert q12.max() <= 1e-5, q12.max()
