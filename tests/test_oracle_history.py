"""Pins of the oracle's history mode (R19).

History mode chains `lookups` lookups per particle through one LCG stream:
the next energy/material are drawn after skipping n_forward = #{c : M_c > 1}
draws.  The pins tie it to things fixed elsewhere:

* P16 (special case = event mode): particle q starts at FF(1070, 10 L q) =
  FF(1070, 2 (5 L q)), so its first lookup IS event lookup 5 L q, which the
  upstream event checksums pin (test_oracle_checksum.py P12).
* P17 (brute force): the chain re-derived in Python with exact integers —
  LCG stepping one draw at a time (no fast-forward), n_forward counted from
  the oracle's own M, materials from the pinned pick rule — must reproduce
  every (p, mat) the oracle reports; and every M must equal the event-mode
  lookup of that (p, mat) (the per-lookup function is the pinned one).
* P18 (invariants): the sum is additive over particle ranges and independent
  of the thread count; v = 1 + argmax M.
"""
import os

import numpy as np
import pytest

import oracle

NT = max(1, min(8, os.cpu_count() or 1))
CONC_SEED = 1070 * 1070
A, C, M63 = 2806196910506780709, 1, 1 << 63


@pytest.fixture(scope="module")
def tiny():
    return oracle.Oracle.from_spec(12, 1000, conc_seed=CONC_SEED, material_rule=1)


@pytest.fixture(scope="module")
def small():
    return oracle.Oracle.from_spec(68, 11303, conc_seed=CONC_SEED, material_rule=0,
                                   hash_bins=8192, nthreads=NT)


@pytest.mark.parametrize("L", [1, 3, 34])
def test_first_lookup_is_event_lookup(tiny, L):
    # P16
    n = 50
    S, out = tiny.run_history(0, n, L, outputs=True)
    for q in range(n):
        r = tiny.lookup(5 * L * q, oracle.UNIONIZED)
        o = q * L
        assert (out["p"][o], out["mat"][o], out["v"][o]) == (r["p"], r["mat"], r["v"])
        assert out["M"][o].tolist() == r["M"].tolist()


def _pick(roll):
    return oracle.pick_mat(roll)


@pytest.mark.parametrize("first", [0, 777])
def test_chain_brute_force(tiny, first):
    # P17 on tiny (n_forward > 0 happens: M_c > 1 for the large materials)
    L, n = 34, 12
    S, out = tiny.run_history(first, n, L, outputs=True)
    nf_seen = set()
    for q in range(n):
        s = 1070
        for _ in range(10 * L * (first + q)):
            s = (A * s + C) % M63
        for i in range(L):
            s = (A * s + C) % M63
            p = s / 2.0**63
            s = (A * s + C) % M63
            mat = _pick(s / 2.0**63)
            o = q * L + i
            assert (out["p"][o], out["mat"][o]) == (p, mat), (q, i)
            Mo = out["M"][o]
            nf = int((Mo > 1.0).sum())
            nf_seen.add(nf)
            for _ in range(nf):
                s = (A * s + C) % M63
    assert len(nf_seen) > 1  # the data dependence is exercised
    # every M is the plain event-mode lookup of its (p, mat)
    S2, M2, v2 = tiny.run_explicit(out["p"], out["mat"], mode=oracle.UNIONIZED)
    assert np.array_equal(M2, out["M"]) and np.array_equal(v2, out["v"])
    assert S == S2 == int(out["v"].sum())


def test_history_invariants(small):
    # P18: additivity over particle ranges, thread-count independence, all
    # grid routes equal (P9 carried over)
    L = 34
    S_all = small.run_history(0, 3000, L, mode=oracle.HASH, nthreads=NT)
    S_a = small.run_history(0, 1234, L, mode=oracle.HASH, nthreads=1)
    S_b = small.run_history(1234, 1766, L, mode=oracle.HASH, nthreads=3)
    assert S_all == S_a + S_b
    assert small.run_history(0, 200, L, mode=oracle.UNIONIZED) == \
        small.run_history(0, 200, L, mode=oracle.HASH) == \
        small.run_history(0, 200, L, mode=oracle.NUCLIDE)
    S, out = small.run_history(5, 40, L, mode=oracle.HASH, outputs=True)
    M = out["M"]
    best = np.full(len(M), -1.0)
    idx = np.zeros(len(M), np.int64)
    for c in range(5):
        upd = M[:, c] > best
        best = np.where(upd, M[:, c], best)
        idx = np.where(upd, c, idx)
    assert np.array_equal(idx + 1, out["v"])
