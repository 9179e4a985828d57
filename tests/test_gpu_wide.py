"""Scorings outside the int8 substitution profile (|p + G_first| > 127;
VERDICT r01 boundary item): the WIDE int32 kernels select p + G_first from
two int32 values by comparing codes, so every scoring inside the SW_ERANGE
rule runs.  Stage 1 (best cell and special rows), the
reverse pass, Stage 2 and the full alignment are compared with the oracle,
which computes in int64 (Eq. 1-3)."""
import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu
WIDE = [(200, -3, 3, 2), (1000, -2000, 500, 100), (5, -300, 200, 1), (100000, -70000, 30000, 1000)]


@pytest.fixture(scope="module")
def ctx():
    from paper_conf_ipps_sandesm11_b200 import Context, build

    build.build()
    c = Context(0)
    yield c
    c.set_grid(0)
    c.close()


def _s(x):
    return x.tobytes().decode() if isinstance(x, np.ndarray) else x


@pytest.mark.parametrize("sc", WIDE)
@pytest.mark.parametrize("m,n,k", [(1, 1, 1), (700, 95, 16), (5000, 2049, 32), (9000, 1500, 7)])
def test_wide_stage1(ctx, sc, m, n, k):
    A, B = synth.random_pair(900 + m + n + sc[0] % 97, m, n, plant_len=min(m, n) // 2, s=0.05, g=0.01)
    got, rows = ctx.align_stage1(A, B, *sc, k=k, keep_rows=True)
    st = ctx.stats()
    assert st["alpha"] > 0  # the int32 kernel
    want, orows = oracle.stage1(_s(A), _s(B), *sc, k=k)
    assert got.astuple() == want
    assert [r for r, _, _ in rows] == [r for r, _, _ in orows]
    for (r, h, f), (_, oh, of) in zip(rows, orows):
        assert np.array_equal(h, oh) and np.array_equal(f, of), r


def test_wide_multiwave(ctx):
    A, B = synth.random_pair(950, 3 * 4096 + 17, 800, plant_len=700, s=0.05, g=0.01)
    ctx.set_grid(2)
    try:
        got, rows = ctx.align_stage1(A, B, *WIDE[1], k=1, keep_rows=True)
    finally:
        ctx.set_grid(0)
    want, orows = oracle.stage1(_s(A), _s(B), *WIDE[1], k=1)
    assert got.astuple() == want
    for (r, h, f), (_, oh, of) in zip(rows, orows):
        assert np.array_equal(h, oh) and np.array_equal(f, of), r


@pytest.mark.parametrize("sc", WIDE)
def test_wide_reverse_stage2_align(ctx, sc):
    A, B = synth.random_pair(960 + sc[1] % 53, 3000, 2600, plant_len=2400, s=0.04, g=0.01)
    want, _ = oracle.stage1(_s(A), _s(B), *sc, k=0)
    best, _ = ctx.align_stage1(A, B, *sc, k=128)
    assert best.astuple() == want
    start = ctx.reverse_goal(A, best.i, B, best.j, best.score, *sc)
    assert start.astuple() == oracle.reverse_goal(_s(A), best.i, _s(B), best.j, *sc, best.score)
    L2 = ctx.stage2(A, B, *sc, k=128, end=best)
    assert L2 == oracle.stage2(_s(A), _s(B), *sc, 128, *want)
    ra = ctx.align(A, B, *sc, k=128)
    wa = oracle.align(_s(A), _s(B), *sc, 128)
    assert (ra["score"], ra["start"], ra["end"]) == (wa["score"], wa["start"], wa["end"])


def test_wide_range_rule(ctx):
    """Scores that could leave the +-2^30 window still fail with SW_ERANGE."""
    from paper_conf_ipps_sandesm11_b200 import SW_ERANGE, SwError

    with pytest.raises(SwError) as e:
        ctx.align_stage1("ACGT" * 3000, "ACGT" * 3000, 100000, -3, 3, 2)
    assert e.value.code == SW_ERANGE
