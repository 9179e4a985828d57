"""The packed 16x2 Stage-1 kernel (N4) forced on, bit-exact against the oracle:
every geometry that has a packed instantiation, special rows (k % 16 == 0),
ragged shapes, several scorings within its value window, virtual stripes,
and the int32 kernel on the same inputs."""
import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu
PAPER = (1, -3, 3, 2)
PACKED_VARIANTS = [0, 1, 3, 5, 6, 8, 9, 10, 11, 12, 13, 14]
# alpha 16: 4, 12, 15 warps + I/O warp, 16 warps with cooperative I/O;
# alpha 32 (16 slots per lane): 4 warps + I/O warp, 4 cooperative, 8 + I/O warp, 16 cooperative, 4 + I/O split F chain


@pytest.fixture(scope="module")
def ctx():
    from paper_conf_ipps_sandesm11_b200 import Context, build

    build.build()
    c = Context(0)
    yield c
    c.set_kernel(-1, True)
    c.set_virtual_stripes(1)
    c.close()


def _s(x):
    return x.tobytes().decode() if isinstance(x, np.ndarray) else x


def check(ctx, A, B, scoring, k, variant, stripes=1, expect_packed=True):
    ctx.set_kernel(variant, True)
    ctx.set_virtual_stripes(stripes)
    try:
        got, rows = ctx.align_stage1(A, B, *scoring, k=k, keep_rows=True)
        st = ctx.stats()
    finally:
        ctx.set_kernel(-1, True)
        ctx.set_virtual_stripes(1)
    assert (st["alpha"] < 0) == expect_packed, st
    # the immediate-patched image runs for every packed geometry but the split-F one (12)
    assert st["patched"] == (1 if expect_packed and variant not in (12,) else 0), st
    want, orows = oracle.stage1(_s(A), _s(B), *scoring, k=k)
    assert got.astuple() == want, (len(A), len(B), scoring, k, variant, stripes)
    assert [r for r, _, _ in rows] == [r for r, _, _ in orows]
    for (r, h, f), (_, oh, of) in zip(rows, orows):
        assert np.array_equal(h, oh), f"H row {r}"
        assert np.array_equal(f, of), f"F row {r}"


@pytest.mark.parametrize("variant", PACKED_VARIANTS)
@pytest.mark.parametrize("m,n", [(1, 1), (17, 1), (16, 300), (1000, 999), (3000, 64), (5000, 2049)])
def test_packed_shapes(ctx, variant, m, n):
    A, B = synth.random_pair(m + 3 * n + variant, m, n, plant_len=min(m, n) // 2, s=0.05, g=0.01)
    check(ctx, A, B, PAPER, 34 if variant == 14 else 32, variant)


@pytest.mark.parametrize("variant", PACKED_VARIANTS)
def test_packed_scorings(ctx, variant):
    A, B = synth.random_pair(5 + variant, 2500, 1700, plant_len=1500, s=0.06, g=0.01)
    for scoring in (PAPER, (2, -1, 4, 1), (1, -1, 0, 2), (5, -4, 10, 1), (3, -2, 0, 1)):
        check(ctx, A, B, scoring, 34 if variant == 14 else 32, variant)
    check(ctx, A, B, PAPER, 0, variant)


def test_packed_falls_back_when_not_applicable(ctx):
    A, B = synth.random_pair(8, 900, 700, plant_len=500)
    check(ctx, A, B, (100, -20, 20, 5), 16, 5, expect_packed=False)  # value window too wide
    check(ctx, A, B, PAPER, 7, 12, expect_packed=False)  # the split-F geometry keeps strip-bottom rows only


ALPHA = {0: 16, 1: 16, 3: 16, 5: 16, 6: 16, 8: 32, 9: 32, 10: 32, 11: 32, 12: 32, 13: 30, 14: 34}
GEN = {0, 1, 8, 10, 13, 14}  # geometries with the generic special-row instantiation


@pytest.mark.parametrize("variant", [0, 1, 5, 8, 10, 13, 14])
@pytest.mark.parametrize("k", [7, 16, 33, 100, 1000, 4097])
def test_packed_any_special_row_interval(ctx, variant, k):
    """Special rows that are not strip bottoms (k >= alpha, not a multiple of
    it): the generic special-row tiles (SPM 2) store the lane's one special row
    from whichever slot and half holds it; every row against the oracle.  k <
    alpha (several rows per lane) runs the int32 kernel."""
    A, B = synth.random_pair(30 + variant + k, 9000, 1300, plant_len=1000, s=0.05, g=0.01)
    check(ctx, A, B, PAPER, k, variant, expect_packed=k % ALPHA[variant] == 0 or (k >= ALPHA[variant] and variant in GEN))


@pytest.mark.parametrize("variant", [0, 10, 13, 14])
def test_packed_staged_special_rows_every_slot(ctx, variant):
    """k >= 32 alpha: one lane per warp holds a special row, which the GEN
    kernel stages in shared memory with its slot as a compile-time constant
    (SPM 3, sw_fill16.cuh tile_gen); k = 32 alpha + d walks the row through
    every slot and both halves of the strip over the matrix, several bands per
    CTA (sw_set_grid 2).  Every special row against the oracle."""
    al = ALPHA[variant]
    for d in (1, al // 2 + 1):
        k = 32 * al + d
        A, B = synth.random_pair(700 + variant + d, 2 * al * k + 77, 530, plant_len=2000, s=0.05, g=0.01)
        ctx.set_grid(2)
        try:
            check(ctx, A, B, PAPER, k, variant, expect_packed=True)
        finally:
            ctx.set_grid(0)


BAND_ROWS = {0: 2048, 8: 4096, 10: 8192, 13: 3840, 14: 8704}


@pytest.mark.parametrize("variant", [0, 8, 10, 13, 14])
def test_packed_band_staged_special_rows(ctx, variant):
    """k >= the band height and not a multiple of alpha: a band holds at most
    one special row, and every warp of that band runs the staged tiles of the
    row's slot (band_sps, sw_fill16.cuh) while only the owning lane stores;
    k = band height + d walks the row over slots, halves and warps, several
    bands per CTA (sw_set_grid 2), the ragged last band included.  Every
    special row against the oracle."""
    al, bh = ALPHA[variant], BAND_ROWS[variant]
    for d in (1, al // 2 + 3, 31 * al + al - 1):
        k = bh + d
        A, B = synth.random_pair(900 + variant + d, 5 * k + 333, 420, plant_len=3000, s=0.05, g=0.01)
        ctx.set_grid(2)
        try:
            check(ctx, A, B, PAPER, k, variant, expect_packed=True)
        finally:
            ctx.set_grid(0)


def test_packed_ties_and_long_alignment(ctx):
    X = synth.random_pair(3, 400, 1)[0]
    XXX = np.concatenate([X, X, X])
    check(ctx, XXX, X, PAPER, 16, 5)
    check(ctx, X, XXX, PAPER, 16, 0)
    A, B = synth.random_pair(21, 9000, 9000, plant_len=9000, s=0.01, g=0.002)  # whole-length: large scores
    check(ctx, A, B, PAPER, 1024, 3)


@pytest.mark.parametrize("stripes", [2, 3, 8])
def test_packed_virtual_stripes(ctx, stripes):
    A, B = synth.random_pair(60 + stripes, 6000, 1500, plant_len=1200, s=0.04, g=0.01)
    check(ctx, A, B, PAPER, 16, 0, stripes=stripes)
    check(ctx, A, B, PAPER, 0, 5, stripes=stripes)


@pytest.mark.parametrize("variant", [8, 9, 10, 11, 12])
def test_packed_alpha32(ctx, variant):
    """16 slots per lane: special rows at strip bottoms (k % 32 == 0), ties,
    stripes, and the int32 fallback when k is only a multiple of 16."""
    A, B = synth.random_pair(70 + variant, 7000, 2100, plant_len=1500, s=0.04, g=0.01)
    check(ctx, A, B, PAPER, 96, variant)
    check(ctx, A, B, (5, -4, 10, 1), 64, variant)
    check(ctx, A, B, PAPER, 16, variant, expect_packed=False)  # k < alpha: two rows per lane, int32
    check(ctx, A, B, PAPER, 48, variant, expect_packed=variant in GEN)  # k % alpha != 0: generic rows (GEN)
    X = synth.random_pair(4, 500, 1)[0]
    check(ctx, np.concatenate([X, X, X, X]), X, PAPER, 32, variant)
    check(ctx, A, B, PAPER, 32, variant, stripes=3)


@pytest.mark.parametrize("m,n", [(1, 1), (29, 40), (31, 300), (3839, 700), (3841, 1000), (9000, 2049)])
def test_packed_alpha30_shapes(ctx, m, n):
    """Variant 13: 15 slots per lane (odd slot count, unpaired last slot) and
    3840-row bands whose strips straddle the 16-code words of A; special rows
    at strip bottoms (k % 30 == 0), bands, ragged tails."""
    A, B = synth.random_pair(130 + m + n, m, n, plant_len=min(m, n) // 2, s=0.05, g=0.01)
    check(ctx, A, B, PAPER, 30, 13)
    check(ctx, A, B, PAPER, 0, 13)


def test_packed_alpha30(ctx):
    A, B = synth.random_pair(131, 8000, 2100, plant_len=1500, s=0.04, g=0.01)
    for scoring in (PAPER, (2, -1, 4, 1), (1, -1, 0, 2), (5, -4, 10, 1), (3, -2, 0, 1)):
        check(ctx, A, B, scoring, 3840, 13)
    check(ctx, A, B, PAPER, 90, 13)
    check(ctx, A, B, PAPER, 32, 13)  # k not a multiple of 30: the GEN instantiation (generic special rows)
    check(ctx, A, B, PAPER, 29, 13, expect_packed=False)  # k < alpha: int32 kernel
    check(ctx, A, B, PAPER, 60, 13, stripes=3)
    X = synth.random_pair(5, 500, 1)[0]
    check(ctx, np.concatenate([X, X, X, X]), X, PAPER, 30, 13)


def test_packed_config_c1(ctx):
    cfg = synth.CONFIGS["C1"]
    A, B = synth.make_pair(cfg)
    check(ctx, A, B, PAPER, cfg.k, 5)


@pytest.mark.parametrize("scoring", [PAPER, (2, -1, 0, 1), (5, -4, 10, 1), (1, -1, 1, 1), (3, -2, 2, 3)])
def test_patch_on_off_identical(ctx, scoring):
    """Patched immediates (per scoring) and register operands give identical
    special rows and best cell, both equal to the oracle."""
    A, B = synth.random_pair(77 + scoring[2], 4000, 3000, plant_len=1500, s=0.03, g=0.01)
    out = []
    for on in (True, False):
        ctx.set_patch(on)
        try:
            got, rows = ctx.align_stage1(A, B, *scoring, k=64, keep_rows=True)
            st = ctx.stats()
        finally:
            ctx.set_patch(True)
        assert st["alpha"] < 0 and st["patched"] == int(on), st
        out.append((got.astuple(), rows))
    assert out[0][0] == out[1][0]
    for (r, h, f), (r2, h2, f2) in zip(out[0][1], out[1][1]):
        assert r == r2 and np.array_equal(h, h2) and np.array_equal(f, f2)
    want, orows = oracle.stage1(_s(A), _s(B), *scoring, k=64)
    assert out[0][0] == want
    for (r, h, f), (_, oh, of) in zip(out[0][1], orows):
        assert np.array_equal(h, oh) and np.array_equal(f, of), r


def test_patch_image_cache_eviction(ctx):
    """More distinct (G_open, G_ext) pairs than the per-context image cache
    holds (4): images are evicted and reloaded, results stay exact."""
    A, B = synth.random_pair(4242, 2500, 2200, plant_len=1200, s=0.04, g=0.01)
    scorings = [(1, -3, 3, 2), (1, -2, 2, 1), (2, -3, 4, 1), (1, -1, 1, 2), (3, -2, 0, 3), (2, -2, 5, 2), (1, -3, 3, 2)]
    for sc in scorings:
        got, rows = ctx.align_stage1(A, B, *sc, k=32, keep_rows=True)
        st = ctx.stats()
        assert st["alpha"] < 0 and st["patched"] == 1, (sc, st)
        want, orows = oracle.stage1(_s(A), _s(B), *sc, k=32)
        assert got.astuple() == want, sc
        for (r, h, f), (_, oh, of) in zip(rows, orows):
            assert np.array_equal(h, oh) and np.array_equal(f, of), (sc, r)
