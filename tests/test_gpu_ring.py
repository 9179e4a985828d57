"""Special rows through a bounded device ring with back-pressure (a6;
VERDICT r01 item 3).

The paper flushes special rows into a bounded Special Rows Area and
Stage 2 reads them back from it.  sw_set_row_budget caps the device
bytes of the ring, so rows wrap around a few slots and every band waits for
its slots until the host has copied the rows that used them before.  Any
k >= 1 must stay bit-exact under any budget: k = 1 dumps the
full H/F matrix through a ring of one band's rows; Stage 2 and the full
alignment then read the rows back from the library's host store.
"""
import time

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
    c.set_row_budget(0)
    c.set_grid(0)
    c.set_kernel(-1, True)
    c.close()


def _s(x):
    return x.tobytes().decode() if isinstance(x, np.ndarray) else x


def run(ctx, A, B, scoring, k, variant=-1, packed=True, grid=0, budget=1, sink=None):
    ctx.set_kernel(variant, packed)
    ctx.set_grid(grid)
    ctx.set_row_budget(budget)
    try:
        got, rows = ctx.align_stage1(A, B, *scoring, k=k, keep_rows=True, sink=sink)
        st = ctx.stats()
    finally:
        ctx.set_kernel(-1, True)
        ctx.set_grid(0)
        ctx.set_row_budget(0)
    return got, rows, st


def compare(got, rows, A, B, scoring, k):
    want, orows = oracle.stage1(_s(A), _s(B), *scoring, k=k)
    assert got.astuple() == want
    assert [r for r, _, _ in rows] == [r for r, _, _ in orows]
    for (r, h, f), (_, oh, of) in zip(rows, orows):
        assert np.array_equal(h, oh), f"H row {r}"
        assert np.array_equal(f, of), f"F row {r}"


@pytest.mark.parametrize("variant,alpha,nw", [(1, 16, 8), (0, 16, 4), (7, 16, 8)])
@pytest.mark.parametrize("grid", [1, 3])
def test_ring_full_matrix_int32(ctx, variant, alpha, nw, grid):
    """k = 1 through the smallest ring (one band's rows + 1): every H and F."""
    bh = alpha * 32 * nw
    m, n = 3 * bh + 211, 777
    A, B = synth.random_pair(6000 + variant + grid, m, n, plant_len=700, s=0.05, g=0.01)
    got, rows, st = run(ctx, A, B, PAPER, 1, variant, False, grid)
    assert st["alpha"] == alpha and 0 < st["sp_slots"] < m, st
    compare(got, rows, A, B, PAPER, 1)


@pytest.mark.parametrize("variant,alpha", [(1, 16), (10, 32), (13, 30), (8, 32)])
def test_ring_packed_strip_rows(ctx, variant, alpha):
    """k = alpha (strip-bottom rows, band bottoms from the I/O warp) and k = 2
    band heights (one row every other band) through a minimal ring."""
    nw = {1: 8, 10: 8, 13: 4, 8: 4}[variant]
    bh = alpha * 32 * nw
    m, n = 5 * bh + 99, 1500
    A, B = synth.random_pair(6100 + variant, m, n, plant_len=1000, s=0.04, g=0.01)
    for k, grid in ((alpha, 2), (2 * bh, 2), (alpha, 0)):
        got, rows, st = run(ctx, A, B, PAPER, k, variant, True, grid)
        assert st["alpha"] == -alpha and (st["sp_slots"] < m // k or k > alpha), st
        compare(got, rows, A, B, PAPER, k)


def test_ring_budget_in_bytes(ctx):
    """A budget of a few rows: the ring holds exactly that many slots (at least
    one band's rows) and the result does not depend on it."""
    A, B = synth.random_pair(6200, 30000, 2000, plant_len=1500, s=0.04, g=0.01)
    k = 512
    slot = 2 * 2016 * 4  # H and F of one row, padded to 32 columns
    for slots in (9, 17, 40):
        got, rows, st = run(ctx, A, B, PAPER, k, budget=slots * slot)
        assert slots <= st["sp_slots"] < 30000 // k, st
        compare(got, rows, A, B, PAPER, k)


def test_ring_slow_sink_back_pressure(ctx):
    """A sink slower than the fill: the kernel must wait for its slots (not
    overwrite rows the host has not copied)."""
    A, B = synth.random_pair(6300, 20000, 3000, plant_len=2000, s=0.04, g=0.01)

    def slow(row, H, F):
        time.sleep(0.002)
        return False

    got, rows, st = run(ctx, A, B, PAPER, 64, 1, True, 2, sink=slow)
    assert st["sp_slots"] < 20000 // 64
    compare(got, rows, A, B, PAPER, 64)


def test_ring_sink_abort_then_reuse(ctx):
    """A sink that aborts while kernels wait on the ring: SW_EABORTED, and the
    context keeps working."""
    from paper_conf_ipps_sandesm11_b200 import SW_EABORTED, SwError

    A, B = synth.random_pair(6400, 20000, 1000, plant_len=800)
    ctx.set_row_budget(1)
    try:
        with pytest.raises(SwError) as ei:
            ctx.align_stage1(A, B, *PAPER, k=16, sink=lambda r, h, f: r >= 160)
        assert ei.value.code == SW_EABORTED
    finally:
        ctx.set_row_budget(0)
    got, rows, st = run(ctx, A, B, PAPER, 16)
    compare(got, rows, A, B, PAPER, 16)


@pytest.mark.parametrize("k", [64, 256, 512])
def test_stage2_from_host_store(ctx, k):
    """Stage 2 reads the special rows back from the host store (the SRA)
    when the ring could not keep them: L_2 identical to the oracle's."""
    A, B = synth.random_pair(6500 + k, 6000, 5000, plant_len=4500, s=0.03, g=0.01)
    ctx.set_row_budget(1)
    try:
        best, _ = ctx.align_stage1(A, B, *PAPER, k=k)
        st = ctx.stats()
        L2 = ctx.stage2(A, B, *PAPER, k=k, end=best)
    finally:
        ctx.set_row_budget(0)
    assert st["sp_slots"] < 6000 // k
    want = oracle.stage2(_s(A), _s(B), *PAPER, k, *best.astuple())
    assert L2 == want


def test_full_alignment_under_ring(ctx):
    """sw_align (Stages 1-5) with a ring that wraps: same score, start and end
    as the oracle's alignment, and the GAP lists rescore to the score."""
    A, B = synth.random_pair(6600, 12000, 11000, plant_len=10000, s=0.03, g=0.01)
    k = 512
    ctx.set_row_budget(1)
    try:
        ra = ctx.align(A, B, *PAPER, k=k)
    finally:
        ctx.set_row_budget(0)
    want = oracle.align(_s(A), _s(B), *PAPER, k)
    assert (ra["score"], ra["start"], ra["end"]) == (want["score"], want["start"], want["end"])
