"""The band pipeline's multi-wave path under oracle parity.

Large configs (C3-C5) have far more bands than resident CTAs, so every CTA
takes several bands from the ticket: per-band re-initialisation, in-place
reuse of the row border, the best carried across bands, special rows of a
later band.  sw_set_grid caps the CTAs of a launch so the same path runs on
inputs the oracle redoes in seconds: bands outnumber CTAs by 2-9x here, with a
ragged last band.  Eq. 1-3 hold for every cell, so the full matrix
(k = 1, int32 kernel) or every strip-bottom row (k = alpha, packed kernel) is
compared with the oracle bit for bit, together with the best cell (P:62,
P:174) and the special rows.
"""
import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu
PAPER = (1, -3, 3, 2)
# (variant, alpha, compute warps) of sw_api.cu variant_for
INT32 = [(0, 16, 4), (1, 16, 8), (2, 8, 8), (3, 16, 12), (4, 16, 14), (5, 16, 15), (6, 16, 16), (7, 16, 8)]
PACKED = [(0, 16, 4), (1, 16, 8), (3, 16, 12), (5, 16, 15), (6, 16, 16), (8, 32, 4), (9, 32, 4), (10, 32, 8),
          (11, 32, 16), (12, 32, 4), (13, 30, 4), (14, 34, 8)]


@pytest.fixture(scope="module")
def ctx():
    from paper_conf_ipps_sandesm11_b200 import Context, build

    build.build()
    c = Context(0)
    yield c
    c.set_grid(0)
    c.set_kernel(-1, True)
    c.set_virtual_stripes(1)
    c.close()


def _s(x):
    return x.tobytes().decode() if isinstance(x, np.ndarray) else x


def run(ctx, A, B, scoring, k, variant, packed, grid, stripes=1):
    ctx.set_kernel(variant, packed)
    ctx.set_grid(grid)
    ctx.set_virtual_stripes(stripes)
    try:
        got, rows = ctx.align_stage1(A, B, *scoring, k=k, keep_rows=True)
        st = ctx.stats()
    finally:
        ctx.set_kernel(-1, True)
        ctx.set_grid(0)
        ctx.set_virtual_stripes(1)
    return got, rows, st


def compare(got, rows, A, B, scoring, k):
    want, orows = oracle.stage1(_s(A), _s(B), *scoring, k=k)
    assert got.astuple() == want
    assert [r for r, _, _ in rows] == [r for r, _, _ in orows]
    for (r, h, f), (_, oh, of) in zip(rows, orows):
        assert np.array_equal(h, oh), f"H row {r}"
        assert np.array_equal(f, of), f"F row {r}"


@pytest.mark.parametrize("variant,alpha,nw", INT32)
@pytest.mark.parametrize("grid", [1, 2, 3])
def test_int32_multiwave_full_matrix(ctx, variant, alpha, nw, grid):
    """k = 1: every H and F of the matrix, with 3-9 bands per CTA."""
    bh = alpha * 32 * nw
    m, n = 2 * bh + bh // 2 + 37, 523
    A, B = synth.random_pair(1000 + 10 * variant + grid, m, n, plant_len=400, s=0.05, g=0.01)
    got, rows, st = run(ctx, A, B, PAPER, 1, variant, False, grid)
    assert st["alpha"] == alpha and st["warps"] == nw and st["grid"] == grid, st
    compare(got, rows, A, B, PAPER, 1)


@pytest.mark.parametrize("variant,alpha,nw", PACKED)
@pytest.mark.parametrize("grid", [1, 2])
def test_packed_multiwave(ctx, variant, alpha, nw, grid):
    """k = alpha: every strip-bottom row (band bottoms drained by the I/O warp
    included), with 3 bands per CTA at grid 1 and a ragged last band."""
    bh = alpha * 32 * nw
    m, n = 2 * bh + bh // 3 + 5, 1111
    A, B = synth.random_pair(2000 + 10 * variant + grid, m, n, plant_len=900, s=0.04, g=0.01)
    got, rows, st = run(ctx, A, B, PAPER, alpha, variant, True, grid)
    assert st["alpha"] == -alpha and st["warps"] == nw and st["grid"] == grid, st
    compare(got, rows, A, B, PAPER, alpha)


@pytest.mark.parametrize("variant,alpha,nw", [(1, 16, 8), (10, 32, 8), (13, 30, 4)])
def test_packed_multiwave_scorings_and_band_rows(ctx, variant, alpha, nw):
    """Special rows at band bottoms only (k = band height) and at a multiple of
    alpha that is not, several scorings, grid 2 over 4+ bands."""
    bh = alpha * 32 * nw
    m, n = 4 * bh + 77, 700
    A, B = synth.random_pair(3000 + variant, m, n, plant_len=600, s=0.05, g=0.01)
    for scoring in (PAPER, (2, -1, 4, 1), (5, -4, 10, 1)):
        for k in (bh, 3 * alpha):
            got, rows, st = run(ctx, A, B, scoring, k, variant, True, 2)
            assert st["alpha"] == -alpha and st["grid"] == 2, st
            compare(got, rows, A, B, scoring, k)


def test_multiwave_best_in_late_band(ctx):
    """The best cell lies in the last (ragged) band and ties occur in earlier
    bands: the best carried across a CTA's bands must keep (max, min i, min j)."""
    X = synth.random_pair(77, 300, 1)[0]
    filler = synth.random_pair(78, 9000, 1)[0]
    A = np.concatenate([X, filler, X, filler[:500], X])  # three equal-scoring copies, in band 0, 2 and the tail
    B = X
    for variant, packed, alpha in ((1, False, 16), (1, True, 16), (10, True, 32)):
        got, rows, st = run(ctx, A, B, PAPER, alpha, variant, packed, 1)
        compare(got, rows, A, B, PAPER, alpha)
        assert got.i == 300  # the first copy wins the tie


@pytest.mark.parametrize("stripes", [2, 3])
def test_multiwave_virtual_stripes(ctx, stripes):
    """Column stripes with several bands per CTA: the per-(band, warp) border
    flags of later bands."""
    m, n = 3 * 4096 + 99, 1800
    A, B = synth.random_pair(4000 + stripes, m, n, plant_len=1200, s=0.04, g=0.01)
    got, rows, st = run(ctx, A, B, PAPER, 1, 1, False, stripes, stripes=stripes)
    assert st["grid"] == stripes, st
    compare(got, rows, A, B, PAPER, 1)
    got, rows, st = run(ctx, A, B, PAPER, 16, 1, True, stripes, stripes=stripes)
    assert st["alpha"] == -16 and st["grid"] == stripes, st
    compare(got, rows, A, B, PAPER, 16)


@pytest.mark.parametrize("variant,packed", [(1, False), (10, True), (0, False)])
def test_reverse_pass_multiwave(ctx, variant, packed):
    """The reverse pass (a8, global mode) over a whole-length alignment: the
    fill spans several bands per CTA and the band with the first hit stops the
    later ones."""
    A, B = synth.random_pair(5000 + variant, 20000, 20000, plant_len=20000, s=0.01, g=0.002)
    want, _ = oracle.stage1(_s(A), _s(B), *PAPER, k=0)
    ctx.set_kernel(variant, packed)
    ctx.set_grid(2)
    try:
        st = ctx.reverse_goal(A, want[1], B, want[2], want[0], *PAPER)
        stats = ctx.stats()
    finally:
        ctx.set_kernel(-1, True)
        ctx.set_grid(0)
    assert stats["grid"] <= 2, stats
    assert st.astuple() == oracle.reverse_goal(_s(A), want[1], _s(B), want[2], *PAPER, want[0])
