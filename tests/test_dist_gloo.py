"""World-size-2 (gloo, CPU) tests of the multi-GPU plumbing: shard ranges,
the A9 all-reduce of the verification vector and the max-over-ranks timing.
The per-shard sums come from the CPU oracle (the CUDA path needs a GPU)."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_sc_tianscd23_b200 import dist as D


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, scaling, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    o = oracle.Oracle.from_spec(12, 1000, conc_seed=1070 * 1070, material_rule=1)
    first, count = D.shard_range(rank, world, 20_000, scaling)
    S = o.run(first, count, nthreads=2)
    vsum = torch.tensor([S, count], dtype=torch.int64)
    D.combine_vsum(vsum)
    tmax = D.max_over_ranks(10.0 + rank)
    q.put((rank, vsum.tolist(), tmax, D.global_hash(vsum)))
    dist.destroy_process_group()


@pytest.mark.parametrize("scaling", ["weak", "strong"])
def test_two_rank_allreduce(scaling):
    import oracle
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, scaling, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = sorted(q.get(timeout=120) for _ in range(world))
    for p in ps:
        p.join(timeout=60)
    o = oracle.Oracle.from_spec(12, 1000, conc_seed=1070 * 1070, material_rule=1)
    total = 20_000 * world if scaling == "weak" else 20_000
    S = o.run(0, total, nthreads=4)
    for rank, vs, tmax, h in res:
        assert vs == [S, total]            # every rank holds the global sum
        assert tmax == 11.0                 # max over ranks
        assert h == S % 999983


def test_shard_ranges_cover_exactly():
    for world in (1, 2, 3, 4, 7, 8):
        L = 17_000_000
        parts = [D.shard_range(r, world, L, "strong") for r in range(world)]
        assert parts[0][0] == 0
        for (a, n), (b, _) in zip(parts, parts[1:]):
            assert a + n == b
        assert sum(n for _, n in parts) == L
        weak = [D.shard_range(r, world, 1000, "weak") for r in range(world)]
        assert weak == [(r * 1000, 1000) for r in range(world)]
    with pytest.raises(ValueError):
        D.shard_range(2, 2, 10)


def _energy_worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import numpy as np

    import oracle
    o = oracle.Oracle.from_spec(12, 1000, conc_seed=1070 * 1070, material_rule=1)
    _, r = o.run(0, 20_000, nthreads=2, outputs=True)
    lo, hi = D.energy_shard_bounds(rank, world)
    sel = (r["p"] >= lo) & (r["p"] < hi)
    vsum = torch.tensor([int(r["v"][sel].sum()), int(sel.sum())], dtype=torch.int64)
    D.combine_vsum(vsum)
    q.put((rank, vsum.tolist(), D.global_hash(vsum)))
    dist.destroy_process_group()


def test_two_rank_energy_shards():
    """Strong scaling by energy ranges (bench.py's multi-GPU default): the
    shards' oracle sums all-reduce to the whole batch's."""
    import oracle
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_energy_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = sorted(q.get(timeout=120) for _ in range(world))
    for p in ps:
        p.join(timeout=60)
    S = oracle.Oracle.from_spec(12, 1000, conc_seed=1070 * 1070, material_rule=1).run(
        0, 20_000, nthreads=4)
    for rank, vs, h in res:
        assert vs == [S, 20_000]
        assert h == S % 999983


def test_energy_shard_bounds_partition():
    """Every energy (including 0, 1, the boundaries and their neighbours)
    falls in exactly one shard, for R in {1, 2, 3, 4, 7, 8}."""
    import numpy as np
    rng = np.random.default_rng(0)
    for R in (1, 2, 3, 4, 7, 8):
        b = [r / R for r in range(1, R)]
        ps = np.concatenate([rng.random(10_000), [0.0, 1.0, -0.5, 1.5], b,
                             np.nextafter(b, 0), np.nextafter(b, 2)])
        hits = np.zeros(ps.size, int)
        for r in range(R):
            lo, hi = D.energy_shard_bounds(r, R)
            hits += (ps >= lo) & (ps < hi)
        assert np.all(hits == 1), R
    with pytest.raises(ValueError):
        D.energy_shard_bounds(3, 3)
