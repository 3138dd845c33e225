"""GPU parity: the CUDA path (through the C-ABI, libxs.so) against the CPU
oracle, element by element on the same seeded inputs.

Bars (BASELINE.json north_star):
  * energy p, material, grid index u/b, bracket k, verification v and the
    hash: bit-exact;
  * macro XS M_c: the kernels accumulate in the oracle's order with no FMA,
    so they are required bit-exact here too (stronger than the 1e-12
    relative bound the north_star allows).
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


@pytest.fixture(scope="module")
def X():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_sc_tianscd23_b200.xs as xs
    return xs


_ORACLES = {}


def oracle_for(name, hash_bins=0):
    key = (name, hash_bins)
    if key not in _ORACLES:
        g = GOLDEN[name]
        _ORACLES[key] = oracle.Oracle.from_spec(g["n_isotopes"], g["n_gridpoints"],
                                                conc_seed=CONC_SEED,
                                                material_rule=g["material_rule"],
                                                hash_bins=hash_bins, nthreads=NT)
    return _ORACLES[key]


def _full_outputs(grid, first, count, **kw):
    want = ("macro_xs", "energy", "mat", "grid_index", "verification")
    vsum, res = grid.lookup(first, count, want=want, **kw)
    torch.cuda.synchronize()
    out = {k: v.cpu().numpy() for k, v in res.items()}
    return [int(x) for x in vsum.cpu()], out


def _compare(out, ref, mode_index=True):
    assert np.array_equal(out["energy"], ref["p"])
    assert np.array_equal(out["mat"], ref["mat"])
    if mode_index:
        assert np.array_equal(out["grid_index"], ref["grid_index"])
    bad = np.nonzero(~np.all(out["macro_xs"] == ref["M"], axis=1))[0]
    assert bad.size == 0, (bad[:10], out["macro_xs"][bad[:3]], ref["M"][bad[:3]])
    assert np.array_equal(out["verification"], ref["v"])


# ------------------------------------------------------------------- tiny --
@pytest.mark.parametrize("variant", ["default", "sort", "baseline", "v1", "v2", "v3", "v4",
                                     "v51", "v52", "v53", "v54",
                                     "sort-v1", "sort-v3", "sort-v4", "sort-v9", "sort-v10",
                                     "sort-v11", "sort-v12", "sort-v17", "sort-v18", "sort-v19",
                                     "sort-v20", "sort-v21", "sort-v22", "sort-v23",
                                     "sort-v24", "sort-v25", "sort-v26", "sort-v27", "sort-v28",
                                     "sort-v40", "sort-v41", "sort-v42", "sort-v43", "sort-v44",
                                     "sort-v45", "sort-v49", "sort-v50", "sort-v55", "sort-v56",
                                     "sort-v57", "sort-v58"])
def test_tiny_full_parity(X, variant):
    g = X.Grid.from_preset("tiny")
    kw = {}
    if variant.startswith("sort"):
        kw["sort"] = True
    if variant == "baseline":
        kw["baseline"] = True
    if variant.startswith("v") or variant.startswith("sort-v"):
        g.set_param("variant", int(variant.split("v")[-1]))
    S, ref = oracle_for("tiny").run(0, 100_000, mode=oracle.UNIONIZED, nthreads=NT, outputs=True)
    vs, out = _full_outputs(g, 0, 100_000, **kw)
    _compare(out, ref)
    assert vs == [S, 100_000]
    assert X.hash_of(vs) == GOLDEN["tiny"]["hash"]


@pytest.mark.parametrize("grid_type,bins", [("hash", 97), ("hash", 8192), ("nuclide", 0)])
@pytest.mark.parametrize("sort", [False, True])
def test_tiny_other_grids(X, grid_type, bins, sort):
    g = X.Grid.from_preset("tiny", grid_type=grid_type, hash_bins=bins)
    mode = oracle.HASH if grid_type == "hash" else oracle.NUCLIDE
    o = oracle_for("tiny", hash_bins=bins)
    S, ref = o.run(0, 100_000, mode=mode, nthreads=NT, outputs=True)
    vs, out = _full_outputs(g, 0, 100_000, sort=sort)
    _compare(out, ref)
    assert vs == [S, 100_000]


@pytest.mark.parametrize("grid_type,bins", [("hash", 97), ("hash", 8192), ("nuclide", 0)])
@pytest.mark.parametrize("variant", [9, 17, 19, 20, 21, 40, 41, 44])
def test_tiny_other_grids_staged(X, grid_type, bins, variant):
    """The TMA-staged sorted gathers on the hash and nuclide grids."""
    g = X.Grid.from_preset("tiny", grid_type=grid_type, hash_bins=bins)
    g.set_param("variant", variant)
    mode = oracle.HASH if grid_type == "hash" else oracle.NUCLIDE
    S, ref = oracle_for("tiny", hash_bins=bins).run(3, 70_001, mode=mode, nthreads=NT,
                                                    outputs=True)
    vs, out = _full_outputs(g, 3, 70_001, sort=True)
    _compare(out, ref)
    assert vs == [S, 70_001]


@pytest.mark.parametrize("layout", ["row", "col", "both"])
@pytest.mark.parametrize("sort", [False, True])
def test_index_layouts(X, layout, sort):
    g = X.Grid.from_preset("tiny", index_layout=layout)
    assert g.info.index_layout == X.INDEX_LAYOUTS[layout]
    S, ref = oracle_for("tiny").run(7, 50_001, mode=oracle.UNIONIZED, nthreads=NT, outputs=True)
    vs, out = _full_outputs(g, 7, 50_001, sort=sort)
    _compare(out, ref)
    assert vs == [S, 50_001]


@pytest.mark.parametrize("first,count", [(0, 1), (5, 7), (123, 31), (999_999, 1001),
                                         (2**31 + 5, 333), (7, 4097), (0, 65_537)])
@pytest.mark.parametrize("variant", [0, 40, 44])
def test_ragged_batches(X, first, count, variant):
    g = X.Grid.from_preset("tiny")
    g.set_param("variant", variant)
    S, ref = oracle_for("tiny").run(first, count, mode=oracle.UNIONIZED, nthreads=NT,
                                    outputs=True)
    for sort in (False, True):
        vs, out = _full_outputs(g, first, count, sort=sort)
        _compare(out, ref)
        assert vs == [S, count]
    # the verification sum alone (the bench's launch: output-free gather
    # instances, next-task energies prefetched; ragged last tasks)
    vsum = torch.zeros(2, dtype=torch.int64, device="cuda")
    g.lookup(first, count, sort=True, vsum=vsum)
    torch.cuda.synchronize()
    assert [int(x) for x in vsum.cpu()] == [S, count]


def test_empty_batch_and_accumulation(X):
    g = X.Grid.from_preset("tiny")
    vsum = torch.tensor([5, 6], dtype=torch.int64, device="cuda")
    g.lookup(0, 0, vsum=vsum)
    g.lookup(0, 1000, vsum=vsum)
    g.lookup(1000, 1000, vsum=vsum)
    torch.cuda.synchronize()
    S = oracle_for("tiny").run(0, 2000, nthreads=NT)
    assert vsum.cpu().tolist() == [S + 5, 2006]


def test_tables_tiny(X):
    g = X.Grid.from_preset("tiny")
    o = oracle_for("tiny")
    assert np.array_equal(g.table(X.XS_TABLE_NUCLIDE_GRID), o.grid().ravel())
    U = g.table(X.XS_TABLE_UNION_ENERGY)
    assert np.array_equal(U, o.union())
    IG = g.table(X.XS_TABLE_INDEX_GRID).reshape(o.NU, o.I)
    ref_ig = o.index_grid_sweep()
    assert np.array_equal(IG, ref_ig)
    assert g.info.index_layout == X.XS_INDEX_BOTH
    IGT = g.table(X.XS_TABLE_INDEX_GRID_T).reshape(o.I, o.NU)
    assert np.array_equal(IGT, ref_ig.T)
    assert np.array_equal(g.table(X.XS_TABLE_MATS).reshape(12, -1), o.mats())
    assert np.array_equal(g.table(X.XS_TABLE_CONCS).reshape(12, -1), o.concs())
    assert np.array_equal(g.table(X.XS_TABLE_NUM_NUCS), o.num_nucs())
    gh = X.Grid.from_preset("tiny", grid_type="hash", hash_bins=257)
    oh = oracle_for("tiny", hash_bins=257)
    HG = gh.table(X.XS_TABLE_INDEX_GRID).reshape(257, 12)
    ref = np.array([[oh.hash_entry(b, n) for n in range(12)] for b in range(257)])
    assert np.array_equal(HG, ref)


@pytest.mark.parametrize("grid_type,bins", [("unionized", 0), ("hash", 64), ("nuclide", 0)])
def test_nuclide_index_edges(X, grid_type, bins):
    g = X.Grid.from_preset("tiny", grid_type=grid_type, hash_bins=bins)
    o = oracle_for("tiny", hash_bins=bins)
    grid = o.grid()
    E = grid[:, :, 0].ravel()
    rng = np.random.default_rng(5)
    probes = np.concatenate([[0.0, 1.0, np.nextafter(1.0, 0), 1e-300], E, np.nextafter(E, 0),
                             np.nextafter(E, 2), np.arange(65) / 64.0, rng.random(5000)])
    nucs = rng.integers(0, 12, probes.size).astype(np.int32)
    k = g.nuclide_index(torch.tensor(probes, device="cuda"),
                        torch.tensor(nucs, device="cuda")).cpu().numpy()
    ref = np.array([o.nuclide_bracket(int(n), float(p)) for p, n in zip(probes, nucs)])
    assert np.array_equal(k, ref)


# ----------------------------------------------------------- explicit API --
def test_explicit_lookups(X):
    g = X.Grid.from_preset("tiny")
    o = oracle_for("tiny")
    rng = np.random.default_rng(11)
    E = o.grid()[:, :, 0].ravel()
    p = np.concatenate([rng.random(20000), E[:500], [0.0, 1.0, -0.25, 1.5, 1e-300]])
    m = rng.integers(0, 12, p.size).astype(np.int32)
    m[7] = 12          # invalid material
    m[11] = -1
    S, M, v = o.run_explicit(np.where((m >= 0) & (m < 12), p, 0.5),
                             np.clip(m, 0, 11), mode=oracle.UNIONIZED, nthreads=NT)
    ok = (m >= 0) & (m < 12)
    for sort in (False, True):
        vs, res = g.lookup_explicit(torch.tensor(p, device="cuda"), torch.tensor(m, device="cuda"),
                                    sort=sort, want=("macro_xs", "verification", "mat"))
        torch.cuda.synchronize()
        Mg = res["macro_xs"].cpu().numpy()
        vg = res["verification"].cpu().numpy()
        assert np.array_equal(Mg[ok], M[ok])
        assert np.array_equal(vg[ok], v[ok])
        assert np.all(vg[~ok] == 0) and np.all(np.isnan(Mg[~ok]))
        assert np.array_equal(res["mat"].cpu().numpy(), m)
        assert vs.cpu().tolist() == [int(v[ok].sum()), int(ok.sum())]
    # host buffers (XS_FLAG_HOST_IO): same results, outputs on the host
    vs, res = g.lookup_explicit(torch.tensor(p), torch.tensor(m), want=("macro_xs",))
    assert np.array_equal(res["macro_xs"].numpy()[ok], M[ok])
    assert vs.tolist() == [int(v[ok].sum()), int(ok.sum())]


def test_verify_entry_point(X):
    g = X.Grid.from_preset("tiny")
    vs, res = g.lookup(0, 5000, want=("macro_xs",))
    v2 = g.verify(res["macro_xs"])
    torch.cuda.synchronize()
    assert vs.cpu().tolist() == v2.cpu().tolist()
    M = torch.tensor([[0.5, 0.5, 0.1, 0.2, 0.3], [-2.0, -3.0, -1.5, -1.0, -4.0],
                      [0.0, 0.0, 0.0, 0.0, 0.0], [1.0, 2.0, 3.0, 4.0, 5.0]], device="cuda",
                     dtype=torch.float64)
    assert g.verify(M).cpu().tolist() == [1 + 1 + 1 + 5, 4]


# --------------------------------------------------- caller-supplied data --
def test_worked_example_through_gpu(X):
    with open(os.path.join(HERE, "golden", "worked_two_nuclide.json")) as f:
        w = json.load(f)
    grid = np.zeros((2, 3, 6))
    for i, name in enumerate(("A", "B")):
        grid[i, :, 0] = w["nuclides"][name]["E"]
        grid[i, :, 1:] = np.array(w["nuclides"][name]["xs"], np.float64)
    for gt, bins in (("unionized", 0), ("hash", 4), ("nuclide", 0)):
        g = X.Grid.from_arrays(grid, [2], [w["material"]["nuclides"]], [w["material"]["concs"]],
                               grid_type=gt, hash_bins=bins)
        p = torch.tensor([c["p"] for c in w["cases"]], device="cuda", dtype=torch.float64)
        m = torch.zeros(len(w["cases"]), dtype=torch.int32, device="cuda")
        vs, res = g.lookup_explicit(p, m, want=("macro_xs", "verification", "grid_index"))
        torch.cuda.synchronize()
        for i, c in enumerate(w["cases"]):
            assert res["macro_xs"][i].cpu().tolist() == c["M"]
            assert int(res["verification"][i]) == c["v"]
            if gt == "unionized":
                assert int(res["grid_index"][i]) == c["u"]


def test_linear_closed_form_at_scale(X):
    # P7 on the GPU with no oracle: dyadic linear channels are interpolated
    # exactly, so M_c = sum_j conc_j (alpha_jc p + beta_jc) for dyadic p.
    rng = np.random.default_rng(2)
    I, N = 40, 200
    E = np.array([np.sort(rng.choice(np.arange(1, 4096), N, replace=False)) for _ in range(I)])
    E = E / 4096.0
    alpha = rng.integers(-8, 9, (I, 5)) / 8.0
    beta = rng.integers(-8, 9, (I, 5)) / 4.0
    grid = np.zeros((I, N, 6))
    grid[:, :, 0] = E
    grid[:, :, 1:] = alpha[:, None, :] * E[:, :, None] + beta[:, None, :]
    mats = np.stack([rng.permutation(I)[:30] for _ in range(3)]).astype(np.int32)
    concs = rng.integers(1, 16, (3, 30)) / 16.0
    g = X.Grid.from_arrays(grid, [30, 30, 30], mats, concs)
    p = rng.integers(0, 4097, 200_000) / 4096.0
    m = rng.integers(0, 3, p.size).astype(np.int32)
    vs, res = g.lookup_explicit(torch.tensor(p, device="cuda"), torch.tensor(m, device="cuda"),
                                want=("macro_xs",))
    got = res["macro_xs"].cpu().numpy()
    ref = np.zeros((p.size, 5))
    for j in range(30):
        n = mats[m, j]
        ref = ref + concs[m, j][:, None] * (alpha[n] * p[:, None] + beta[n])
    assert np.array_equal(got, ref)


def test_invalid_arguments(X):
    with pytest.raises(X.XSError) as e:
        X.Grid.from_spec(n_isotopes=100, n_gridpoints=100, material_rule=0)
    assert e.value.status == 1
    with pytest.raises(X.XSError):
        X.Grid.from_spec(n_isotopes=12, n_gridpoints=1, material_rule=1)
    g = X.Grid.from_preset("tiny")
    vsum = torch.zeros(2, dtype=torch.int64, device="cuda")
    o = X.xs_outputs(None, None, None, None, None, vsum.data_ptr())
    with pytest.raises(X.XSError):  # workspace too small
        X.xs_lookup_batch(g._h, 0, 1000, 0, o, g.workspace(10).data_ptr(), 16,
                          torch.cuda.current_stream().cuda_stream)
    with pytest.raises(X.XSError):  # unknown flag
        X.xs_lookup_batch(g._h, 0, 10, 0x80, o, g.workspace(10).data_ptr(), 1 << 20,
                          torch.cuda.current_stream().cuda_stream)
    bad = np.zeros((1, 3, 6))
    bad[0, :, 0] = [0.1, 0.1, 0.2]   # duplicate energy
    with pytest.raises(X.XSError) as e:
        X.Grid.from_arrays(bad, [1], [[0]], [[1.0]])
    assert e.value.status == 6


# ------------------------------------------------------ full-size configs --
def _sample_ids(L, k=3000, seed=0):
    rng = np.random.default_rng(seed)
    ids = np.concatenate([[0, 1, L - 1, L // 2], rng.integers(0, L, k)])
    return np.unique(ids)


@pytest.mark.parametrize("name", ["small", "large", "large-hash", "xl"])
def test_full_config_hash_and_samples(X, name):
    gold = GOLDEN[name]
    if name == "xl":
        free, _ = torch.cuda.mem_get_info()
        if free < 140e9:
            pytest.skip("XL needs ~130 GB of device memory")
    g = X.Grid.from_preset(name)
    pre = X.PRESETS[name]
    L = pre["lookups"]
    sort = pre.get("sort", False)
    # the launch configuration bench.py times: one batch of all L lookups
    if L <= 20_000_000:
        want = ("energy", "mat", "grid_index", "verification")
        vs, res = g.lookup(0, L, sort=sort, want=want)
        torch.cuda.synchronize()
        assert [int(x) for x in vs.cpu()] == [gold["sum_v"], L]
        ids = _sample_ids(L)
        o = oracle_for(name, hash_bins=pre.get("hash_bins", 0))
        mode = oracle.HASH if pre["grid_type"] == "hash" else oracle.UNIONIZED
        ids_t = torch.tensor(ids, device="cuda")
        E = res["energy"][ids_t].cpu().numpy()
        mt = res["mat"][ids_t].cpu().numpy()
        gi = res["grid_index"][ids_t].cpu().numpy()
        v = res["verification"][ids_t].cpu().numpy()
        # macro XS for the sampled ids through the explicit entry point
        _, rex = g.lookup_explicit(torch.tensor(E, device="cuda"), torch.tensor(mt, device="cuda"),
                                   want=("macro_xs",))
        Mx = rex["macro_xs"].cpu().numpy()
        for j, i in enumerate(ids):
            r = o.lookup(int(i), mode)
            assert (E[j], mt[j], gi[j], v[j]) == (r["p"], r["mat"], r["grid_index"], r["v"]), i
            assert np.array_equal(Mx[j], r["M"]), i
    else:
        # XL: 170M lookups in 10 shards of 17M (the bench's per-GPU batch size)
        vsum = torch.zeros(2, dtype=torch.int64, device="cuda")
        step = 17_000_000
        for first in range(0, L, step):
            g.lookup(first, min(step, L - first), vsum=vsum)
        torch.cuda.synchronize()
        assert [int(x) for x in vsum.cpu()] == [gold["sum_v"], L]
        ids = _sample_ids(L, k=400)
        o = oracle_for("xl", hash_bins=131072)
        for i in ids:
            i = int(i)
            vs, res = g.lookup(i, 1, want=("energy", "mat", "grid_index", "macro_xs",
                                           "verification"))
            r = o.lookup(i, oracle.HASH)
            assert float(res["energy"][0]) == r["p"] and int(res["mat"][0]) == r["mat"]
            assert int(res["grid_index"][0]) == o.union_index(r["p"])
            assert res["macro_xs"][0].cpu().tolist() == r["M"].tolist()
            assert int(res["verification"][0]) == r["v"]
    assert X.hash_of([gold["sum_v"]]) == gold["hash"]


def test_shard_invariance_small(X):
    # P10: sum over contiguous shards == one batch, for R in {1,2,3,4,7,8}
    g = X.Grid.from_preset("small")
    L = 17_000_000
    sums = []
    for R in (1, 2, 3, 4, 7, 8):
        vsum = torch.zeros(2, dtype=torch.int64, device="cuda")
        for r in range(R):
            a, b = r * L // R, (r + 1) * L // R
            g.lookup(a, b - a, vsum=vsum, sort=(R % 2 == 0))
        torch.cuda.synchronize()
        sums.append(vsum.cpu().tolist())
    assert all(s == [GOLDEN["small"]["sum_v"], L] for s in sums)


def test_bench_multirank_path_on_one_gpu(X):
    """bench.py's N > 1 path (shards, barrier, max-over-ranks, A9 all-reduce)
    with two ranks sharing the box's GPU over gloo."""
    import subprocess
    import sys
    root = os.path.dirname(HERE)
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
                        "--nproc-per-node", "2", "--master-addr", "127.0.0.1", "--master-port",
                        "29541", "bench.py", "--gpus", "2", "--backend", "gloo", "--config", "small",
                        "--scaling", "weak",
                        "--steps", "3", "--warmup", "3", "--no-cpu-baseline", "--no-e2e"],
                       cwd=root, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["lookups_per_step"] == 2 * 17_000_000
    # ids [0, 34M): rank 0's shard is the golden small batch; the global sum
    # must equal the oracle's over both shards
    assert d["hash"] == (GOLDEN["small"]["sum_v"] + _small_second_shard_sum()) % 999983


def test_bench_strong_energy_shards_on_one_gpu(X):
    """bench.py's default multi-GPU mode (strong scaling, energy-range
    shards) with two gloo ranks sharing the GPU, self-launched by
    `bench.py --gpus 2` (no torchrun on the command line): the global
    verification sum is the one-batch golden sum."""
    import subprocess
    import sys
    root = os.path.dirname(HERE)
    r = subprocess.run([sys.executable, "bench.py", "--gpus", "2", "--backend", "gloo",
                        "--config", "small", "--steps", "3", "--warmup", "3",
                        "--no-cpu-baseline", "--e2e-steps", "1"],
                       cwd=root, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["scaling"] == "strong"
    assert d["lookups_per_step"] == 17_000_000
    assert d["hash"] == GOLDEN["small"]["hash"] and d["hash_matches_oracle"] is True
    assert d["e2e"]["vsum_matches_batch"] is True
    assert d["a9_allreduce_ms_per_step"] > 0


def _small_second_shard_sum():
    o = oracle.Oracle.from_spec(68, 11303, conc_seed=CONC_SEED, material_rule=0, hash_bins=8192,
                                nthreads=NT)
    return o.run(17_000_000, 17_000_000, mode=oracle.HASH, nthreads=NT)


@pytest.mark.parametrize("sort", [False, True])
def test_explicit_host_io_chunked(X, sort):
    # XS_FLAG_HOST_IO inputs larger than host_chunk are uploaded and looked up
    # chunk by chunk (overlapped); results must not depend on the chunking
    g = X.Grid.from_preset("tiny")
    o = oracle_for("tiny")
    rng = np.random.default_rng(21)
    p = rng.random(50_003)
    m = rng.integers(0, 12, p.size).astype(np.int32)
    S, M, v = o.run_explicit(p, m, mode=oracle.UNIONIZED, nthreads=NT)
    for chunk, mt in [(1 << 22, m), (7_001, m), (1_024, m), (7_001, m.astype(np.uint8))]:
        g.set_param("host_chunk", chunk)
        vs, res = g.lookup_explicit(torch.tensor(p), torch.tensor(mt), sort=sort,
                                    want=("macro_xs", "verification"))
        assert vs.tolist() == [S, p.size]
        assert np.array_equal(res["macro_xs"].numpy(), M)
        assert np.array_equal(res["verification"].numpy(), v)


@pytest.mark.parametrize("variant", [0, 9, 17, 19, 20, 21, 25, 28, 40, 41, 42, 43, 44, 45, 49,
                                     50, 55, 56, 57, 58])
@pytest.mark.parametrize("grid_type,bins", [("unionized", 0), ("hash", 97)])
def test_vsum_only_sorted(X, variant, grid_type, bins):
    """Sorted batches with only vsum requested (no per-lookup outputs: the
    staged gathers search U only at each task's extreme energies)."""
    g = X.Grid.from_preset("tiny", grid_type=grid_type, hash_bins=bins)
    g.set_param("variant", variant)
    mode = oracle.HASH if grid_type == "hash" else oracle.UNIONIZED
    for first, count in [(0, 100_000), (77, 4099), (5, 1)]:
        S = oracle_for("tiny", hash_bins=bins).run(first, count, mode=mode, nthreads=NT)
        vs, _ = g.lookup(first, count, sort=True)
        torch.cuda.synchronize()
        assert [int(x) for x in vs.cpu()] == [S, count]


@pytest.mark.parametrize("host", [False, True])
@pytest.mark.parametrize("sort", [False, True])
def test_explicit_lookups_u8_materials(X, host, sort):
    """XS_FLAG_MAT_U8: one byte per material id, same results as int32 ids;
    ids >= n_mats (e.g. 255) are invalid lookups."""
    g = X.Grid.from_preset("tiny")
    o = oracle_for("tiny")
    rng = np.random.default_rng(21)
    p = rng.random(30_001)
    m = rng.integers(0, 12, p.size).astype(np.uint8)
    m[3] = 255
    m[9] = 12
    ok = m < 12
    S, M, v = o.run_explicit(np.where(ok, p, 0.5), np.where(ok, m, 0).astype(np.int32),
                             mode=oracle.UNIONIZED, nthreads=NT)
    dev = "cpu" if host else "cuda"
    vs, res = g.lookup_explicit(torch.tensor(p, device=dev), torch.tensor(m, device=dev),
                                sort=sort, want=("macro_xs", "verification", "mat"))
    torch.cuda.synchronize()
    Mg, vg = res["macro_xs"].cpu().numpy(), res["verification"].cpu().numpy()
    assert np.array_equal(Mg[ok], M[ok]) and np.array_equal(vg[ok], v[ok])
    assert np.all(vg[~ok] == 0)
    assert np.array_equal(res["mat"].cpu().numpy(), m.astype(np.int32))
    assert [int(x) for x in vs.cpu()] == [int(v[ok].sum()), int(ok.sum())]


def test_explicit_host_io_unchunked_large(X):
    """Regression: a 17M-lookup sorted batch uploaded in one chunk.  The
    partitioned A2's tile histograms (2076 tiles x 1664 keys) are larger than
    the global-atomic bin array; the workspace must reserve the larger of the
    two (they used to overflow into the staged host inputs)."""
    g = X.Grid.from_preset("large")
    L = GOLDEN["large"]["lookups"]
    vs0, res = g.lookup(0, L, sort=True, want=("energy", "mat"))
    torch.cuda.synchronize()
    assert int(vs0[0]) == GOLDEN["large"]["sum_v"]
    e = res["energy"].cpu().pin_memory()
    m = res["mat"].cpu().to(torch.uint8).pin_memory()
    g.set_param("host_chunk", L)
    vs = torch.zeros(2, dtype=torch.int64).pin_memory()
    g.lookup_explicit(e, m, sort=True, vsum=vs)
    assert [int(x) for x in vs] == [GOLDEN["large"]["sum_v"], L]
    g.close()


def test_sorted_batch_above_48m(X):
    """A sorted batch of more than 48M lookups (partitioned A2 with more than
    4000 tiles) equals the unsorted batch, per lookup and in the sum."""
    g = X.Grid.from_preset("small")
    L = 48_000_000 + 4_321
    vs_s, rs_ = g.lookup(7, L, sort=True, want=("verification",))
    vs_u, ru = g.lookup(7, L, sort=False, want=("verification",))
    torch.cuda.synchronize()
    assert [int(x) for x in vs_s.cpu()] == [int(x) for x in vs_u.cpu()]
    assert int(vs_s[1]) == L
    assert torch.equal(rs_["verification"], ru["verification"])
    g.close()


@pytest.mark.parametrize("sort", [False, True])
def test_explicit_gate_both_kernels_agree(X, sort):
    """Explicit energies run as a gated pair (k_check_energies): a batch of
    safe energies takes the unchecked gather, the same batch plus one energy
    below 2^-440 takes the range-checked one; both equal the oracle."""
    g = X.Grid.from_preset("tiny")
    o = oracle_for("tiny")
    rng = np.random.default_rng(5)
    p = rng.random(50_000)
    m = rng.integers(0, 12, p.size).astype(np.int32)
    S, M, v = o.run_explicit(p, m, mode=oracle.UNIONIZED, nthreads=NT)
    for extra in ([], [2.0 ** -450]):
        pp = np.concatenate([p, extra])
        mm = np.concatenate([m, np.zeros(len(extra), np.int32)])
        vs, res = g.lookup_explicit(torch.tensor(pp, device="cuda"), torch.tensor(mm, device="cuda"),
                                    sort=sort, want=("macro_xs",))
        torch.cuda.synchronize()
        assert np.array_equal(res["macro_xs"].cpu().numpy()[:p.size], M)
        if not extra:
            assert vs.cpu().tolist() == [S, p.size]
    g.close()


@pytest.mark.gpu
@pytest.mark.parametrize("fine_cap", [0, 2048])
@pytest.mark.parametrize("fine_direct", [0, 2, 1024])
@pytest.mark.parametrize("cbits", [6, 7, 8, 9])
def test_part_cbits_tiny_parity(X, cbits, fine_direct, fine_cap):
    """Every coarse fan-out of the partitioned A2 (part_cbits 6-9), with the
    fine pass windowed or scattering directly (fine_direct 0: every segment),
    gives the oracle's per-lookup results; the order inside the sort never
    matters."""
    g = X.Grid.from_preset("tiny")
    g.set_param("part_cbits", cbits)
    g.set_param("fine_direct", fine_direct)
    g.set_param("fine_cap", fine_cap)  # 2048: many windows per segment
    S, ref = oracle_for("tiny").run(3, 100_000, mode=oracle.UNIONIZED, nthreads=NT, outputs=True)
    vs, out = _full_outputs(g, 3, 100_000, sort=True)
    _compare(out, ref)
    assert vs == [S, 100_000]


@pytest.mark.gpu
def test_part_cbits_wide_above_2p26(X):
    """A batch above 2^26 lookups sorted with the widest coarse key
    (part_cbits 9, 53 MB more tile histograms) agrees, per lookup, with the
    default (7)."""
    g = X.Grid.from_preset("small")
    L = (1 << 26) + 12_345
    g.set_param("part_cbits", 9)
    vs_a, ra = g.lookup(11, L, sort=True, want=("verification",))
    g.set_param("part_cbits", 7)
    vs_7, r7 = g.lookup(11, L, sort=True, want=("verification",))
    torch.cuda.synchronize()
    assert [int(x) for x in vs_a.cpu()] == [int(x) for x in vs_7.cpu()]
    assert int(vs_a[1]) == L
    assert torch.equal(ra["verification"], r7["verification"])
    g.close()


@pytest.mark.parametrize("sort", [False, True])
def test_explicit_host_async_pipelined(X, sort):
    """XS_FLAG_HOST_ASYNC: consecutive calls on two alternating workspaces
    (upload of one overlapping the lookups of the other) give each call's
    own results; nothing is read before the stream is synchronized."""
    g = X.Grid.from_preset("tiny")
    o = oracle_for("tiny")
    rng = np.random.default_rng(33)
    batches = []
    for k in range(5):
        p = rng.random(40_000 + 1_000 * k)
        m = rng.integers(0, 12, p.size).astype(np.uint8)
        S, M, v = o.run_explicit(p, m.astype(np.int32), mode=oracle.UNIONIZED, nthreads=NT)
        batches.append((torch.tensor(p).pin_memory(), torch.tensor(m).pin_memory(), S, M, v))
    fl = (X.XS_FLAG_SORT if sort else 0) | X.XS_FLAG_HOST_ASYNC | X.XS_FLAG_MAT_U8
    n = g.workspace_size(45_000, fl)
    wss = [torch.empty(n, dtype=torch.uint8, device="cuda") for _ in range(2)]
    outs = []
    for k, (pt, mt, *_rest) in enumerate(batches):
        vs = torch.zeros(2, dtype=torch.int64).pin_memory()
        _, res = g.lookup_explicit(pt, mt, sort=sort, vsum=vs, want=("macro_xs", "verification"),
                                   asynchronous=True, workspace=wss[k % 2])
        outs.append((vs, res))
    torch.cuda.synchronize()
    for (pt, mt, S, M, v), (vs, res) in zip(batches, outs):
        assert vs.tolist() == [S, pt.numel()]
        assert np.array_equal(res["macro_xs"].numpy(), M)
        assert np.array_equal(res["verification"].numpy(), v)
    with pytest.raises(X.XSError):   # exclusive with XS_FLAG_HOST_IO
        X.xs_lookup_explicit(g._h, batches[0][0].data_ptr(), batches[0][1].data_ptr(), 10,
                             X.XS_FLAG_HOST_IO | X.XS_FLAG_HOST_ASYNC | X.XS_FLAG_MAT_U8,
                             X.xs_outputs(None, None, None, None, None, outs[0][0].data_ptr()),
                             wss[0].data_ptr(), wss[0].numel(), torch.cuda.current_stream().cuda_stream)
