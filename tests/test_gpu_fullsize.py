"""Full-size GPU parity of the headline path (VERDICT r01 "what's missing" #1,
#4): the energy-sorted batch exactly as bench.py times it
(A2 partitioned sort + the staged gather k_gather_s3 with the variant the
density picks), every lookup compared with the CPU oracle; the device-built
tables compared with the oracle's at full size; energy-range shards (the
multi-GPU strong-scaling partition) against the single batch.

Bars (north_star): p, material, grid index, v and the verification sum
bit-exact; M bit-exact (R17: the kernels keep the oracle's
operation order, so bit-exact is required, stronger than 1e-12 relative).
"""
import json
import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import oracle  # noqa: E402

HERE = os.path.dirname(os.path.abspath(__file__))
NT = max(1, min(32, os.cpu_count() or 1))
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


def _oracle(name, hash_bins):
    g = GOLDEN[name]
    return oracle.Oracle.from_spec(g["n_isotopes"], g["n_gridpoints"], conc_seed=CONC_SEED,
                                   material_rule=g["material_rule"], hash_bins=hash_bins,
                                   nthreads=NT)


def _mode(X, name):
    return oracle.HASH if X.PRESETS[name]["grid_type"] == "hash" else oracle.UNIONIZED


def _assert_equal(name, got, ref):
    if not np.array_equal(got, ref):
        eq = (got == ref).reshape(len(got), -1)
        bad = np.nonzero(~np.all(eq, axis=1))[0]
        raise AssertionError(f"{name}: {bad.size} mismatches, first ids {bad[:8]}: "
                             f"{got[bad[:3]]} vs {ref[bad[:3]]}")


# ------------------------------------------- sorted batch, every lookup --
@pytest.mark.parametrize("name", ["small", "large", "large-hash"])
def test_sorted_batch_every_lookup(X, name):
    """All 17M lookups of the sorted batch (sort=True, default variant chosen
    by density: k_gather_s3 variant 25 at this size) against the oracle."""
    gold = GOLDEN[name]
    L = gold["lookups"]
    pre = X.PRESETS[name]
    g = X.Grid.from_preset(name)
    vs, res = g.lookup(0, L, sort=True, want=WANT)
    torch.cuda.synchronize()
    out = {k: v.cpu().numpy() for k, v in res.items()}
    del res
    g.close()
    o = _oracle(name, pre.get("hash_bins", 0))
    S, ref = o.run(0, L, mode=_mode(X, name), nthreads=NT, outputs=True)
    assert S == gold["sum_v"]
    _assert_equal("energy", out["energy"], ref["p"])
    _assert_equal("mat", out["mat"], ref["mat"])
    _assert_equal("grid_index", out["grid_index"], ref["grid_index"])
    _assert_equal("macro_xs", out["macro_xs"], ref["M"])
    _assert_equal("verification", out["verification"], ref["v"])
    assert [int(x) for x in vs.cpu()] == [S, L]


def test_sorted_xl_sampled_million(X):
    """XL: the 170M-lookup sorted batch in one call (bench's launch), 1M
    lookup ids (100 blocks of 10,000 at seeded offsets) compared with the
    oracle element by element, and the verification sum of all 170M."""
    free, _ = torch.cuda.mem_get_info()
    if free < 150e9:
        pytest.skip("XL sorted batch with per-lookup outputs needs ~145 GB of device memory")
    gold = GOLDEN["xl"]
    L = gold["lookups"]
    g = X.Grid.from_preset("xl")
    vs, res = g.lookup(0, L, sort=True, want=("macro_xs", "energy", "mat", "verification"))
    torch.cuda.synchronize()
    assert [int(x) for x in vs.cpu()] == [gold["sum_v"], L]
    rng = np.random.default_rng(17)
    starts = np.sort(rng.choice(L // 10_000, 100, replace=False)) * 10_000
    ids = np.concatenate([np.arange(s, s + 10_000) for s in starts])
    ids_t = torch.tensor(ids, device="cuda")
    out = {k: v[ids_t].cpu().numpy() for k, v in res.items()}
    del res
    g.close()
    o = oracle.Oracle.from_spec(355, 238847, conc_seed=CONC_SEED, material_rule=0,
                                hash_bins=131072, nthreads=NT)
    for b, s in enumerate(starts):
        _, ref = o.run(int(s), 10_000, mode=oracle.HASH, nthreads=NT, outputs=True)
        sl = slice(b * 10_000, (b + 1) * 10_000)
        _assert_equal(f"energy@{s}", out["energy"][sl], ref["p"])
        _assert_equal(f"mat@{s}", out["mat"][sl], ref["mat"])
        _assert_equal(f"macro_xs@{s}", out["macro_xs"][sl], ref["M"])
        _assert_equal(f"verification@{s}", out["verification"][sl], ref["v"])


# --------------------------------------------------- device-built tables --
@pytest.mark.parametrize("name", ["small", "large"])
def test_device_tables_full(X, name):
    """U, IG (row layout), IGT (column layout), the interval tables (K0d,
    K0e) built on the device equal their definitions computed by the oracle
    (R6; DESIGN.md §4 K0d/K0e), every entry."""
    g = X.Grid.from_preset(name, index_layout="both")
    o = _oracle(name, 0)
    I, N, NU = o.I, o.N, o.NU
    _assert_equal("U", g.table(X.XS_TABLE_UNION_ENERGY), o.union())
    grid = o.grid()
    _assert_equal("nuclide grid", g.table(X.XS_TABLE_NUCLIDE_GRID).reshape(I, N, 6), grid)
    step = 1 << 20
    for e0 in range(0, NU, step):
        e1 = min(NU, e0 + step)
        ref = o.index_grid_rows(e0, e1)
        dev = g.table(X.XS_TABLE_INDEX_GRID, e0 * I, (e1 - e0) * I).reshape(e1 - e0, I)
        _assert_equal(f"IG rows {e0}..{e1}", dev, ref)
        for n in range(I):
            col = g.table(X.XS_TABLE_INDEX_GRID_T, n * NU + e0, e1 - e0)
            _assert_equal(f"IGT[{n}] {e0}..{e1}", col, ref[:, n])
    # interval table K0d: {E[k+1], gap, r, 0, (hi.c, hi.c - lo.c) x 5}
    iv = g.table(X.XS_TABLE_INTERVALS).reshape(I, N, 14)
    lo, hi = grid[:, :-1], grid[:, 1:]
    _assert_equal("IV E", iv[:, :-1, 0], hi[..., 0])
    gap = hi[..., 0] - lo[..., 0]
    _assert_equal("IV gap", iv[:, :-1, 1], gap)
    # the reciprocal serves the correctly rounded division; its definition is
    # 1/gap to within the refinement's accuracy
    assert np.max(np.abs(iv[:, :-1, 2] * gap - 1.0)) < 2.0 ** -50
    _assert_equal("IV hi", iv[:, :-1, 4::2], hi[..., 1:])
    _assert_equal("IV d", iv[:, :-1, 5::2], hi[..., 1:] - lo[..., 1:])
    assert not np.any(iv[:, -1]) and not np.any(iv[:, :, 3])
    # K0u (unsorted gather): {E[k+1], gap, (hi.c, hi.c - lo.c) x 5}, 96 B
    ivu = g.table(X.XS_TABLE_INTERVALS_U).reshape(I, N, 12)
    _assert_equal("IVU head", ivu[:, :, :2], iv[:, :, :2])
    _assert_equal("IVU channels", ivu[:, :, 2:], iv[:, :, 4:])
    # fp32 table K0e: h = RN32(hi.c), d = RN32(h - RN32(lo.c)) (R18)
    iv32 = g.table(X.XS_TABLE_INTERVALS32).reshape(I, N, 10)
    _assert_equal("IV32 head", iv32[:, :-1, :3], iv[:, :-1, :3])
    f = iv32[:, :-1, 4:].copy().view(np.float32).reshape(I, N - 1, 12)
    h32 = hi[..., 1:].astype(np.float32)
    _assert_equal("IV32 h", f[..., 0:10:2], h32)
    _assert_equal("IV32 d", f[..., 1:10:2], h32 - lo[..., 1:].astype(np.float32))
    g.close()


def test_device_hash_grid_full(X):
    """HG of large-hash (8,192 bins x 355 nuclides) = R7's definition."""
    g = X.Grid.from_preset("large-hash")
    o = _oracle("large-hash", 8192)
    dev = g.table(X.XS_TABLE_INDEX_GRID).reshape(8192, 355)
    _assert_equal("HG", dev, o.hash_grid(8192))
    g.close()


def test_device_tables_xl_sampled_rows(X):
    """XL: U in full; IGT (120 GB, column layout) on 64 random windows of
    4,096 consecutive unionized energies for every nuclide."""
    free, _ = torch.cuda.mem_get_info()
    if free < 140e9:
        pytest.skip("XL needs ~130 GB of device memory")
    g = X.Grid.from_preset("xl")
    o = oracle.Oracle.from_spec(355, 238847, conc_seed=CONC_SEED, material_rule=0, nthreads=NT)
    NU, I = o.NU, o.I
    _assert_equal("U", g.table(X.XS_TABLE_UNION_ENERGY), o.union())
    rng = np.random.default_rng(3)
    starts = np.concatenate([[0, NU - 4096], rng.integers(0, NU - 4096, 62)])
    for e0 in starts:
        e0 = int(e0)
        ref = o.index_grid_rows(e0, e0 + 4096)
        for n in range(I):
            col = g.table(X.XS_TABLE_INDEX_GRID_T, n * NU + e0, 4096)
            _assert_equal(f"IGT[{n}] {e0}", col, ref[:, n])
    g.close()


# ------------------------------------------------- energy-range shards --
@pytest.mark.parametrize("R", [1, 2, 3, 4, 7, 8])
def test_energy_shards_tiny_every_lookup(X, R):
    """xs_lookup_batch_shard: the R shards of one batch fill every output
    position exactly once and equal the oracle's per-lookup results; shard
    r looks up exactly the lookups with b_r <= p < b_{r+1}."""
    g = X.Grid.from_preset("tiny")
    L, first = 100_000, 11
    S, ref = _oracle("tiny", 0).run(first, L, mode=oracle.UNIONIZED, nthreads=NT, outputs=True)
    _, outs = g.lookup_shard(first, L, 0, R, want=WANT)   # allocates the outputs
    torch.cuda.synchronize()
    for t in outs.values():   # poison: every position must be written by its shard
        t.fill_(float("nan") if t.dtype == torch.float64 else -7)
    total = [0, 0]
    b = [-np.inf] + [r / R for r in range(1, R)] + [np.inf]
    for r in range(R):
        vs = torch.zeros(2, dtype=torch.int64, device="cuda")
        g.lookup_shard(first, L, r, R, vsum=vs, outputs=outs)
        torch.cuda.synchronize()
        sel = (ref["p"] >= b[r]) & (ref["p"] < b[r + 1])
        n_in, v_in = int(np.count_nonzero(sel)), int(ref["v"][sel].sum())
        assert [int(x) for x in vs.cpu()] == [v_in, n_in]
        total[0] += v_in
        total[1] += n_in
    assert total == [S, L]
    out = {k: v.cpu().numpy() for k, v in outs.items()}
    _assert_equal("energy", out["energy"], ref["p"])
    _assert_equal("mat", out["mat"], ref["mat"])
    _assert_equal("grid_index", out["grid_index"], ref["grid_index"])
    _assert_equal("macro_xs", out["macro_xs"], ref["M"])
    _assert_equal("verification", out["verification"], ref["v"])


def test_energy_shards_p10_small(X):
    """P10 with the strong-scaling partition: the shards of the 17M small
    batch sum to the oracle's verification sum for R in {1, 2, 3, 4, 7, 8}."""
    g = X.Grid.from_preset("small")
    L = 17_000_000
    for R in (1, 2, 3, 4, 7, 8):
        vsum = torch.zeros(2, dtype=torch.int64, device="cuda")
        for r in range(R):
            g.lookup_shard(0, L, r, R, vsum=vsum)
        torch.cuda.synchronize()
        assert [int(x) for x in vsum.cpu()] == [GOLDEN["small"]["sum_v"], L], R


def test_energy_shards_large_f32_and_hash(X):
    """Shards with the fp32 variant and on the hash grid (large sizes)."""
    L = 17_000_000
    for name, f32, key in (("large", True, "sum_v_f32"), ("large-hash", False, "sum_v")):
        g = X.Grid.from_preset(name)
        vsum = torch.zeros(2, dtype=torch.int64, device="cuda")
        for r in range(8):
            g.lookup_shard(0, L, r, 8, vsum=vsum, f32=f32)
        torch.cuda.synchronize()
        assert [int(x) for x in vsum.cpu()] == [GOLDEN[name][key], L], name
        g.close()


@pytest.mark.parametrize("R,tiles,cbits", [(8, 1, 0), (8, 16, 0), (3, 2, 8), (8, 0, 8), (32, 0, 0)])
def test_energy_shard_tiles_and_keys(X, R, tiles, cbits):
    """The shard A2 knobs (tile-length factor, coarse key bits) never change
    results: R shards of the 17M small batch sum to the oracle's verification
    sum (R = 32 lengthens the tiles 16-fold), and the shards of a tiny batch
    reproduce every lookup."""
    g = X.Grid.from_preset("small")
    g.set_param("shard_tiles", tiles)
    g.set_param("part_cbits", cbits)
    L = 17_000_000
    vsum = torch.zeros(2, dtype=torch.int64, device="cuda")
    for r in range(R):
        g.lookup_shard(0, L, r, R, vsum=vsum)
    torch.cuda.synchronize()
    assert [int(x) for x in vsum.cpu()] == [GOLDEN["small"]["sum_v"], L]
    g.close()
    g = X.Grid.from_preset("tiny")
    g.set_param("shard_tiles", tiles)
    g.set_param("part_cbits", cbits)
    L, first = 100_000, 5
    S, ref = _oracle("tiny", 0).run(first, L, mode=oracle.UNIONIZED, nthreads=NT, outputs=True)
    _, outs = g.lookup_shard(first, L, 0, R, want=("macro_xs", "verification"))
    total = torch.zeros(2, dtype=torch.int64, device="cuda")
    for r in range(R):
        g.lookup_shard(first, L, r, R, vsum=total, outputs=outs)
    torch.cuda.synchronize()
    assert [int(x) for x in total.cpu()] == [S, L]
    _assert_equal("macro_xs", outs["macro_xs"].cpu().numpy(), ref["M"])
    _assert_equal("verification", outs["verification"].cpu().numpy(), ref["v"])
    with pytest.raises(X.XSError):
        g.set_param("shard_tiles", 17)


def test_energy_shards_xl(X):
    """XL, the north_star's 8-GPU configuration: the 8 energy-range shards of
    the 170M batch (the launch bench.py's projection times; its shards take
    the longer tiles and the extra coarse key bit) sum to the oracle's
    verification sum."""
    free, _ = torch.cuda.mem_get_info()
    if free < 140e9:
        pytest.skip("XL needs ~130 GB of device memory")
    gold = GOLDEN["xl"]
    L = gold["lookups"]
    g = X.Grid.from_preset("xl")
    vsum = torch.zeros(2, dtype=torch.int64, device="cuda")
    for r in range(8):
        g.lookup_shard(0, L, r, 8, vsum=vsum)
    torch.cuda.synchronize()
    assert [int(x) for x in vsum.cpu()] == [gold["sum_v"], L]
    g.close()


def test_energy_shard_arguments(X):
    g = X.Grid.from_preset("tiny")
    vsum = torch.zeros(2, dtype=torch.int64, device="cuda")
    ws = g.workspace(1000, X.XS_FLAG_SORT)
    o = X.xs_outputs(None, None, None, None, None, vsum.data_ptr())
    st = torch.cuda.current_stream().cuda_stream
    for shard, R, flags in ((2, 2, X.XS_FLAG_SORT), (-1, 2, X.XS_FLAG_SORT), (0, 0, X.XS_FLAG_SORT),
                            (0, 2, 0), (0, 2, X.XS_FLAG_SORT | X.XS_FLAG_BASELINE)):
        with pytest.raises(X.XSError) as e:
            X.xs_lookup_batch_shard(g._h, 0, 1000, shard, R, flags, o, ws.data_ptr(), ws.numel(), st)
        assert e.value.status == 1
    g.set_param("legacy_sort", 1)   # no partitioned A2 -> unsupported
    with pytest.raises(X.XSError) as e:
        X.xs_lookup_batch_shard(g._h, 0, 1000, 0, 2, X.XS_FLAG_SORT, o, ws.data_ptr(), ws.numel(),
                                st)
    assert e.value.status == 4


# ------------------------------------------ A2 fine pass: skewed inputs --
@pytest.mark.parametrize("fine_cap", [2048, 0])
def test_fine_pass_clustered_energies(X, fine_cap):
    """Explicit lookups clustered in energy: one material's
    50k lookups in [0.5, 0.5 + 2^-12) make one coarse-key segment longer
    than the fine pass's window (multi-window loop, fine_cap 2048 -> 1365
    lookups with positions), and 3,000 equal energies make one fine bin
    larger than the window (the in-place branch)."""
    g = X.Grid.from_preset("tiny")
    g.set_param("fine_cap", fine_cap)
    g.set_param("fine_direct", 1024)   # windowed, never the direct scatter
    o = _oracle("tiny", 0)
    rng = np.random.default_rng(8)
    p = np.concatenate([0.5 + rng.random(50_000) * 2.0 ** -12, np.full(3_000, 0.25),
                        rng.random(20_000)])
    m = np.concatenate([np.full(50_000, 3), np.full(3_000, 3),
                        rng.integers(0, 12, 20_000)]).astype(np.int32)
    S, M, v = o.run_explicit(p, m, mode=oracle.UNIONIZED, nthreads=NT)
    vs, res = g.lookup_explicit(torch.tensor(p, device="cuda"), torch.tensor(m, device="cuda"),
                                sort=True, want=("macro_xs", "verification"))
    torch.cuda.synchronize()
    _assert_equal("macro_xs", res["macro_xs"].cpu().numpy(), M)
    _assert_equal("verification", res["verification"].cpu().numpy(), v)
    assert [int(x) for x in vs.cpu()] == [S, p.size]


def test_chunked_host_batch_wide_key_fits_workspace(X):
    """a chunked host-input batch whose chunks allow a
    wider coarse key than the whole batch (part_cbits 9: 336M lookups do not
    fit 9 bits, 168M-lookup chunks do) must not write its tile histograms
    past the workspace's bin area; the sum equals the oracle's."""
    import psutil
    if psutil.virtual_memory().available < 48e9:
        pytest.skip("needs ~40 GB of host memory")
    free, _ = torch.cuda.mem_get_info()
    if free < 40e9:
        pytest.skip("needs ~30 GB of device memory")
    L = 336_000_000
    g = X.Grid.from_preset("tiny")
    g.set_param("part_cbits", 9)
    g.set_param("host_chunk", L // 2)
    rng = np.random.default_rng(1)
    p = rng.random(L)
    m = rng.integers(0, 12, L).astype(np.uint8)
    S = _oracle("tiny", 0).run_explicit(p, m.astype(np.int32), mode=oracle.UNIONIZED,
                                        nthreads=NT, outputs=False)
    pt = torch.from_numpy(p).pin_memory()
    mt = torch.from_numpy(m).pin_memory()
    vs, _ = g.lookup_explicit(pt, mt, sort=True)
    assert [int(x) for x in vs] == [S, L]
    g.close()
