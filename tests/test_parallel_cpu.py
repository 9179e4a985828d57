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


# ---------------------------------------------------------------- group logic with a stand-in context

class FakeCtx:
    """Stands in for the library context on CPU: records what the groups ask
    for (handles, epochs, plans) and returns a per-rank local best."""

    def __init__(self, rank, epoch0, plan=(-32, 8)):
        self.rank, self.epoch0, self._plan = rank, epoch0, plan
        self.calls, self.connected = [], None

    # band-cyclic
    def cyclic_export(self, max_rows, max_cols):
        return bytes([100 + self.rank]) * 64

    def cyclic_connect(self, h, max_rows, max_cols):
        self.connected = h

    def cyclic_epoch(self):
        return self.epoch0 + len(self.calls)

    def plan(self, m, n, *sc, k=0, world=0):
        return self._plan

    def align_stage1_cyclic(self, dA, m, dB, n, rank, world, epoch, *sc, k=0, sink=None, stream=0):
        from paper_conf_ipps_sandesm11_b200 import Result

        self.calls.append(epoch)
        return Result(7, 10 + (rank % 2), 3), []

    # column stripes
    def stripe_export(self, max_rows):
        return bytes([self.rank]) * 64

    def stripe_connect(self, h, max_rows):
        self.connected = h

    def stripe_epoch(self):
        return self.epoch0 + len(self.calls)

    def align_stage1_stripe(self, dA, m, dB, n, c_lo, c_hi, epoch, *sc, k=0, sink=None, stream=0):
        from paper_conf_ipps_sandesm11_b200 import Result

        self.calls.append(epoch)
        return Result(7, 20 - self.rank, c_lo + 1), []


def _group_worker(rank, world, port, q, kind):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_ipps_sandesm11_b200.parallel import CyclicGroup, StripeGroup

        ctx = FakeCtx(rank, epoch0=5 * rank)  # contexts that ran different numbers of calls before
        if kind == "cyclic":
            g = CyclicGroup(ctx, rank, world, max_rows=100, max_cols=100)
            res = [g.align_stage1(0, 50, 0, 60)[0] for _ in range(2)]
        else:
            g = StripeGroup(ctx, rank, world, max_rows=100)
            res = [g.align_stage1(0, 50, 0, 60)[0] for _ in range(2)]
        q.put((rank, ctx.connected, ctx.calls, res))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("kind", ["cyclic", "stripes"])
@pytest.mark.parametrize("world", [2, 3])
def test_groups_agree_on_epoch_and_best(kind, world):
    """Handles go to the right neighbour (cyclic: (r + 1) mod world), every rank
    runs each call with the same epoch, above every rank's previous one (the
    flags / progress tags of reused areas), and the combined best agrees."""
    port = 31500 + random.randint(0, 2000)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_group_worker, args=(r, world, port, q, kind)) for r in range(world)]
    for p in procs:
        p.start()
    out = {}
    for _ in range(world):
        rank, conn, calls, res = q.get(timeout=120)
        out[rank] = (conn, calls, res)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    epochs = {tuple(out[r][1]) for r in range(world)}
    assert len(epochs) == 1
    e = epochs.pop()
    assert e[0] > 5 * (world - 1) and e[1] > e[0]
    for r in range(world):
        if kind == "cyclic":
            assert out[r][0] == bytes([100 + (r + 1) % world]) * 64
        else:
            assert out[r][0] == (bytes([r + 1]) * 64 if r + 1 < world else None)
    bests = {tuple(map(tuple, out[r][2])) for r in range(world)}
    assert len(bests) == 1
    if kind == "cyclic":
        assert bests.pop()[0] == (7, 10, 3)
    else:
        assert bests.pop()[0] == (7, 20 - (world - 1), (60 * (world - 1)) // world + 1)
