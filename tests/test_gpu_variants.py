"""Every fixed geometry of the int32 band kernel (sw_set_kernel(v, 0)),
bit-exact against the oracle: ragged shapes, several scorings, special rows
at strip-bottom (k % 16 == 0) and arbitrary rows, virtual stripes, and the
reverse-goal pass (GLOBAL instantiation).  The automatic choice only picks
some of these; the others are tuning points and must be equally exact."""
import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu
PAPER = (1, -3, 3, 2)
INT32_VARIANTS = list(range(8))  # (alpha, warps, W) per sw_api.cu variant_for


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


def check(ctx, A, B, scoring, k, variant, stripes=1):
    ctx.set_kernel(variant, False)
    ctx.set_virtual_stripes(stripes)
    try:
        got, rows = ctx.align_stage1(A, B, *scoring, k=k, keep_rows=True)
        st = ctx.stats()
    finally:
        ctx.set_kernel(-1, True)
        ctx.set_virtual_stripes(1)
    assert st["alpha"] > 0, st
    want, orows = oracle.stage1(_s(A), _s(B), *scoring, k=k)
    assert got.astuple() == want, (len(A), len(B), scoring, k, variant, stripes)
    assert [r for r, _, _ in rows] == [r for r, _, _ in orows]
    for (r, h, f), (_, oh, of) in zip(rows, orows):
        assert np.array_equal(h, oh), f"H row {r}"
        assert np.array_equal(f, of), f"F row {r}"


@pytest.mark.parametrize("variant", INT32_VARIANTS)
@pytest.mark.parametrize("m,n", [(1, 1), (31, 2), (700, 95), (4100, 3001)])
def test_variant_shapes(ctx, variant, m, n):
    A, B = synth.random_pair(7 * m + n + variant, m, n, plant_len=min(m, n) // 2, s=0.05, g=0.01)
    check(ctx, A, B, PAPER, 16, variant)


@pytest.mark.parametrize("variant", INT32_VARIANTS)
def test_variant_scorings_and_rows(ctx, variant):
    A, B = synth.random_pair(50 + variant, 2600, 1900, plant_len=1500, s=0.06, g=0.01)
    for scoring, k in ((PAPER, 7), ((2, -1, 4, 1), 32), ((1, -1, 0, 2), 0), ((100, -20, 20, 5), 100)):
        check(ctx, A, B, scoring, k, variant)


@pytest.mark.parametrize("variant", INT32_VARIANTS)
def test_variant_stripes(ctx, variant):
    A, B = synth.random_pair(90 + variant, 3000, 2500, plant_len=2000, s=0.04, g=0.01)
    check(ctx, A, B, PAPER, 48, variant, stripes=3)


@pytest.mark.parametrize("variant", INT32_VARIANTS)
def test_variant_reverse_goal(ctx, variant):
    A, B = synth.random_pair(130 + variant, 3000, 2800, plant_len=2500, s=0.03, g=0.01)
    (s, ie, je), _ = oracle.stage1(_s(A), _s(B), *PAPER, k=0)
    want = oracle.reverse_goal(_s(A), ie, _s(B), je, *PAPER, s)
    ctx.set_kernel(variant, False)
    try:
        got = ctx.reverse_goal(A, ie, B, je, s, *PAPER)
    finally:
        ctx.set_kernel(-1, True)
    assert got.astuple() == want
