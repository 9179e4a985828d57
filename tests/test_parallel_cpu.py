"""Host-side logic of the multi-GPU column-stripe pipeline, on CPU (gloo,
world size 2): partitioning, the best-cell order across ranks, and the
receive-area handle exchange."""
import os
import random

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_sandesm11_b200.parallel import combine_best, exchange_handles, stripe_bounds


def test_stripe_bounds_partition():
    for n in (8, 9, 100, 536165, 46_944_323):
        for world in (1, 2, 3, 4, 8):
            if n < world:
                continue
            b = [stripe_bounds(n, world, r) for r in range(world)]
            assert b[0][0] == 0 and b[-1][1] == n
            assert all(b[r][1] == b[r + 1][0] for r in range(world - 1))
            assert all(hi > lo for lo, hi in b)
            widths = [hi - lo for lo, hi in b]
            assert max(widths) - min(widths) <= 1
    with pytest.raises(ValueError):
        stripe_bounds(3, 4, 0)


def test_combine_best_order():
    rng = random.Random(1)
    for _ in range(200):
        res = [(rng.randint(0, 5), rng.randint(0, 9), rng.randint(0, 9)) for _ in range(rng.randint(1, 8))]
        pos = [r for r in res if r[0] > 0]
        want = (0, 0, 0) if not pos else min(pos, key=lambda x: (-x[0], x[1], x[2]))
        assert combine_best(res) == want


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        mine = bytes([rank]) * 64 if rank > 0 else None  # rank 0 has no left neighbour
        right = exchange_handles(mine, rank, world)
        lo, hi = stripe_bounds(1000, world, rank)
        local = (10 + (rank % 2), 5 + rank, lo + 1)  # equal scores across ranks exercise the tie-break
        allres = [None] * world
        dist.all_gather_object(allres, local)
        q.put((rank, right, (lo, hi), combine_best(allres)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_gloo_handle_exchange_and_best(world):
    port = 29500 + random.randint(0, 2000)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = {}
    for _ in range(world):
        rank, right, bounds, best = q.get(timeout=120)
        out[rank] = (right, bounds, best)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for r in range(world):
        right, bounds, best = out[r]
        assert right == (bytes([r + 1]) * 64 if r + 1 < world else None)
        assert bounds == stripe_bounds(1000, world, r)
    bests = {out[r][2] for r in range(world)}
    assert len(bests) == 1  # every rank agrees
    # odd ranks score 11; the smallest such rank has the smallest i
    assert bests.pop()[0] == 11
