"""The column-stripe border protocol on the GPU, bit-exact against the oracle
and against the single-stripe run: virtual stripes in one launch (the same
kernel code path as one stripe per GPU), and two processes sharing one GPU
through CUDA IPC (the multi-GPU host path)."""
import os
import random

import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu
PAPER = (1, -3, 3, 2)


@pytest.fixture(scope="module")
def ctx():
    from paper_conf_ipps_sandesm11_b200 import Context, build

    build.build()
    c = Context(0)
    yield c
    c.set_virtual_stripes(1)
    c.close()


def _s(x):
    return x.tobytes().decode() if isinstance(x, np.ndarray) else x


def check(ctx, A, B, scoring, k, stripes):
    ctx.set_virtual_stripes(stripes)
    try:
        got, rows = ctx.align_stage1(A, B, *scoring, k=k, keep_rows=True)
    finally:
        ctx.set_virtual_stripes(1)
    want, orows = oracle.stage1(_s(A), _s(B), *scoring, k=k)
    assert got.astuple() == want, (len(A), len(B), stripes)
    assert [r for r, _, _ in rows] == [r for r, _, _ in orows]
    for (r, h, f), (_, oh, of) in zip(rows, orows):
        assert np.array_equal(h, oh), f"H row {r} stripes={stripes}"
        assert np.array_equal(f, of), f"F row {r} stripes={stripes}"


@pytest.mark.parametrize("stripes", [2, 3, 4, 8])
def test_virtual_stripes_full_matrix(ctx, stripes):
    A, B = synth.random_pair(40 + stripes, 1500, 1200, plant_len=900, s=0.05, g=0.01)
    check(ctx, A, B, PAPER, 1, stripes)


@pytest.mark.parametrize("stripes", [2, 5, 8])
def test_virtual_stripes_narrow_and_ragged(ctx, stripes):
    # stripes narrower than a tile (n / stripes < 64) and ragged widths
    for n in (stripes * 7 + 3, 97, 333):
        if n < stripes:
            continue
        A, B = synth.random_pair(n, 5000, n, plant_len=min(n, 300))
        check(ctx, A, B, PAPER, 64, stripes)


def test_virtual_stripes_many_bands_and_scorings(ctx):
    A, B = synth.random_pair(7, 20000, 3001, plant_len=2500, s=0.03, g=0.005)
    for scoring in (PAPER, (2, -1, 4, 1), (1, -1, 0, 2)):
        check(ctx, A, B, scoring, 4096, 4)
    check(ctx, A, B, PAPER, 1000, 3)  # k not a multiple of alpha


def test_virtual_stripes_ties_across_borders(ctx):
    X = synth.random_pair(3, 400, 1)[0]
    XXX = np.concatenate([X, X, X])
    check(ctx, X, XXX, PAPER, 1, 3)  # equal maxima in different stripes: the first column wins
    check(ctx, XXX, X, PAPER, 1, 2)


def test_virtual_stripes_config_c1(ctx):
    cfg = synth.CONFIGS["C1"]
    A, B = synth.make_pair(cfg)
    check(ctx, A, B, PAPER, cfg.k, 4)


# ---------------------------------------------------------------- two processes, one GPU, CUDA IPC

def _rank_main(rank, world, port, A, B, k, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_sandesm11_b200 import Context
    from paper_conf_ipps_sandesm11_b200.parallel import StripeGroup

    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        ctx = Context(0)
        dA = torch.from_numpy(A).cuda()
        dB = torch.from_numpy(B).cuda()
        grp = StripeGroup(ctx, rank, world, max_rows=len(A))
        rows = {}

        def sink(row, H, F):
            rows[row] = (H.copy(), F.copy())

        res = []
        for _ in range(2):  # two alignments: epochs 1 and 2 reuse the border areas
            best, local, bounds = grp.align_stage1(dA.data_ptr(), len(A), dB.data_ptr(), len(B), PAPER, k=k, sink=sink)
            res.append(best)
        # a second group on the same context: its receive area still
        # holds the first group's flags; the agreed epoch must be above them
        grp2 = StripeGroup(ctx, rank, world, max_rows=len(A))
        best, local, bounds = grp2.align_stage1(dA.data_ptr(), len(A), dB.data_ptr(), len(B), PAPER, k=k, sink=sink)
        res.append(best)
        q.put((rank, res, bounds, rows))
        ctx.close()
    except Exception as e:  # report instead of hanging the parent
        q.put((rank, repr(e), None, None))
    finally:
        dist.destroy_process_group()


def test_two_ranks_ipc_one_gpu():
    import torch.multiprocessing as mp

    A, B = synth.random_pair(11, 9000, 2500, plant_len=2000, s=0.04, g=0.01)
    k = 1024
    world = 2
    port = 31000 + random.randint(0, 2000)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    env = dict(os.environ, SWB_TIMEOUT_S="60")
    os.environ["SWB_TIMEOUT_S"] = "60"
    procs = [ctx.Process(target=_rank_main, args=(r, world, port, A, B, k, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = {}
    for _ in range(world):
        rank, res, bounds, rows = q.get(timeout=300)
        got[rank] = (res, bounds, rows)
    for p in procs:
        p.join(timeout=60)
    for r in range(world):
        assert not isinstance(got[r][0], str), got[r][0]
    want, orows = oracle.stage1(_s(A), _s(B), *PAPER, k=k)
    for r in range(world):
        assert got[r][0] == [want, want, want]
    for row, oh, of in orows:
        h = np.concatenate([got[r][2][row][0] for r in range(world)])
        f = np.concatenate([got[r][2][row][1] for r in range(world)])
        assert np.array_equal(h, oh) and np.array_equal(f, of), row


# ---------------------------------------------------------------- band-cyclic ranks, one GPU, CUDA IPC

def _cyc_rank_main(rank, world, port, A, B, k, q, variant=1):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_sandesm11_b200 import Context
    from paper_conf_ipps_sandesm11_b200.parallel import CyclicGroup

    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        ctx = Context(0)
        ctx.set_kernel(variant, True)  # 4096-row (1) or 8704-row (14) bands: several per rank
        ctx.set_grid(2)          # the two processes time-share one GPU: keep their CTAs few
        dA = torch.from_numpy(A).cuda()
        dB = torch.from_numpy(B).cuda()
        rows = {}

        def sink(row, H, F):
            rows[row] = (H.copy(), F.copy())

        res = []
        for _ in range(2):  # two groups on one context: epochs agreed above the areas' old tags
            grp = CyclicGroup(ctx, rank, world, max_rows=len(A), max_cols=len(B))
            best, local = grp.align_stage1(dA.data_ptr(), len(A), dB.data_ptr(), len(B), PAPER, k=k, sink=sink)
            res.append(best)
        q.put((rank, res, rows))
        ctx.close()
    except Exception as e:  # report instead of hanging the parent
        q.put((rank, repr(e), None))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("variant,bh,k", [(1, 4096, 512), (14, 8704, 8704 + 5)])
def test_two_cyclic_ranks_ipc_one_gpu(variant, bh, k):
    """Band-cyclic ranks in two processes (CUDA IPC areas): every special row
    comes from exactly one rank, whole, bit-exact; the combined best is the
    oracle's.  Variant 14 (alpha 34, the geometry band-cyclic C4 runs on
    several GPUs) with special rows inside the bands (the staged GEN tiles)."""
    import torch.multiprocessing as mp

    A, B = synth.random_pair(12 + variant, 4 * bh + 1234, 1900, plant_len=1500, s=0.04, g=0.01)
    world = 2
    port = 33000 + random.randint(0, 2000)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    os.environ["SWB_TIMEOUT_S"] = "60"
    procs = [ctx.Process(target=_cyc_rank_main, args=(r, world, port, A, B, k, q, variant)) for r in range(world)]
    for p in procs:
        p.start()
    got = {}
    for _ in range(world):
        rank, res, rows = q.get(timeout=300)
        got[rank] = (res, rows)
    for p in procs:
        p.join(timeout=60)
    for r in range(world):
        assert not isinstance(got[r][0], str), got[r][0]
    want, orows = oracle.stage1(_s(A), _s(B), *PAPER, k=k)
    for r in range(world):
        assert got[r][0] == [want, want]
    assert set(got[0][1]).isdisjoint(got[1][1])
    allrows = {**got[0][1], **got[1][1]}
    assert sorted(allrows) == [r for r, _, _ in orows]
    for row, oh, of in orows:
        h, f = allrows[row]
        assert np.array_equal(h, oh) and np.array_equal(f, of), row
