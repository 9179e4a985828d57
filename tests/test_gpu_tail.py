"""The tail segment of a multi-wave fill.

When the bands of a fill leave a partial last wave (C4: 1221 bands of 8192
rows on 148 CTAs), the rows after the last full wave run as a second launch
with a shorter band height that continues the first launch's row border and
band progress.  Eq. 1-3 hold for every cell whichever launch
computes it: every special row, the best cell and the rows at the
segment boundary are compared with the oracle bit for bit.
"""
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
    c.set_tail(-1)
    c.set_grid(0)
    c.set_kernel(-1, True)
    c.close()


def _s(x):
    return x.tobytes().decode() if isinstance(x, np.ndarray) else x


def compare(got, rows, A, B, scoring, k):
    want, orows = oracle.stage1(_s(A), _s(B), *scoring, k=k)
    assert got.astuple() == want
    assert [r for r, _, _ in rows] == [r for r, _, _ in orows]
    for (r, h, f), (_, oh, of) in zip(rows, orows):
        assert np.array_equal(h, oh), f"H row {r}"
        assert np.array_equal(f, of), f"F row {r}"


# (main variant, alpha, warps) x (tail variant, alpha, warps): every tail geometry shorter than the main band
PAIRS = [((10, 32, 8), (0, 16, 4)), ((10, 32, 8), (13, 30, 4)), ((10, 32, 8), (8, 32, 4)), ((10, 32, 8), (1, 16, 8)),
         ((1, 16, 8), (0, 16, 4)), ((13, 30, 4), (0, 16, 4)), ((5, 16, 15), (1, 16, 8))]


@pytest.mark.parametrize("main,tail", PAIRS)
@pytest.mark.parametrize("grid", [2, 3])
def test_forced_tail(ctx, main, tail, grid):
    """grid CTAs, 2 grid + 1 bands: two full waves, then the tail rows in the
    tail geometry (several tail bands per CTA at this grid)."""
    (v, a, w), (vt, at, wt) = main, tail
    bh = a * 32 * w
    m, n = (2 * grid) * bh + bh // 2 + 45, 1300
    A, B = synth.random_pair(7000 + 17 * v + vt + grid, m, n, plant_len=1000, s=0.04, g=0.01)
    # special rows every strip of both geometries, and at the segment boundary
    k = int(np.lcm(a, at))
    ctx.set_kernel(v, True)
    ctx.set_tail(vt + 1)
    ctx.set_grid(grid)
    try:
        got, rows = ctx.align_stage1(A, B, *PAPER, k=k, keep_rows=True)
        st = ctx.stats()
    finally:
        ctx.set_kernel(-1, True)
        ctx.set_tail(-1)
        ctx.set_grid(0)
    assert (st["alpha"], st["warps"], st["grid"]) == (-a, w, grid), st
    assert (st["tail_alpha"], st["tail_warps"]) == (-at, wt), st
    assert st["tail_rows"] == m - 2 * grid * bh and 0 < st["tail_grid"] <= grid, st
    compare(got, rows, A, B, PAPER, k)


def test_tail_best_cell_at_segment_boundary(ctx):
    """Equal best cells, one alignment straddling the segment boundary (its end
    in the tail launch) and a later copy: the (max, min i, min j) order across
    the two launches' slots."""
    v, a, w = 10, 32, 8
    bh = a * 32 * w
    X = synth.random_pair(7100, 500, 1)[0]
    fill = synth.random_pair(7101, 4 * bh, 1)[0]
    A = np.concatenate([fill[: 4 * bh - 250], X, fill[:300], X])  # 4 bh + 1050 rows: 5 bands, grid 2 -> tail after 4
    ctx.set_kernel(v, True)
    ctx.set_tail(1)  # variant 0 (alpha 16, 4 warps)
    ctx.set_grid(2)
    try:
        got, rows = ctx.align_stage1(A, X, *PAPER, k=32, keep_rows=True)
        st = ctx.stats()
    finally:
        ctx.set_kernel(-1, True)
        ctx.set_tail(-1)
        ctx.set_grid(0)
    assert st["tail_alpha"] == -16 and st["tail_rows"] == 1050, st
    compare(got, rows, A, X, PAPER, 32)
    assert got.i == 4 * bh + 250


def test_tail_not_used_when_not_qualifying(ctx):
    """k not a multiple of the tail's alpha, whole waves only, or one wave: no tail."""
    A, B = synth.random_pair(7200, 5 * 8192 + 10, 700, plant_len=500)
    ctx.set_kernel(10, True)
    ctx.set_grid(2)
    try:
        ctx.set_tail(14)  # variant 13 (alpha 30)
        got, rows = ctx.align_stage1(A, B, *PAPER, k=32, keep_rows=True)
        assert ctx.stats()["tail_alpha"] == 0
        compare(got, rows, A, B, PAPER, 32)
        ctx.set_grid(6)  # one wave
        ctx.set_tail(1)
        got, rows = ctx.align_stage1(A, B, *PAPER, k=32, keep_rows=True)
        assert ctx.stats()["tail_alpha"] == 0
    finally:
        ctx.set_kernel(-1, True)
        ctx.set_tail(-1)
        ctx.set_grid(0)
