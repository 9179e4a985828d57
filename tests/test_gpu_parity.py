"""GPU parity: the sm_100a path (through the C ABI) against the CPU oracle on
the same seeded inputs.  Integer results must be bit-exact: best score, end
cell, every special row of H and F, and the reverse-pass start cell."""
import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu

PAPER = (1, -3, 3, 2)
SCORINGS = [PAPER, (2, -1, 4, 1), (1, -1, 0, 2), (5, -4, 10, 1), (3, -2, 0, 1), (100, -20, 20, 5)]


@pytest.fixture(scope="module")
def ctx():
    from paper_conf_ipps_sandesm11_b200 import Context, build

    build.build()
    c = Context(0)
    yield c
    c.close()


def _s(x):
    return x.tobytes().decode() if isinstance(x, np.ndarray) else x


def check_stage1(ctx, A, B, scoring, k):
    got, rows = ctx.align_stage1(A, B, *scoring, k=k, keep_rows=True)
    want, orows = oracle.stage1(_s(A), _s(B), *scoring, k=k)
    assert got.astuple() == want, (len(A), len(B), scoring, k)
    assert [r for r, _, _ in rows] == [r for r, _, _ in orows]
    for (r, h, f), (_, oh, of) in zip(rows, orows):
        assert np.array_equal(h, oh), f"H row {r}"
        assert np.array_equal(f, of), f"F row {r}"
    return got


@pytest.mark.parametrize("m,n", [(1, 1), (1, 97), (97, 1), (31, 32), (32, 33), (33, 31), (200, 200), (1000, 3000), (3000, 1000)])
def test_small_shapes_full_matrix(ctx, m, n):
    """k = 1 dumps every row: the whole H and F matrices are compared."""
    A, B = synth.random_pair(m * 7 + n, m, n, plant_len=min(m, n) // 2)
    check_stage1(ctx, A, B, PAPER, 1)


@pytest.mark.parametrize("scoring", SCORINGS)
def test_scorings_full_matrix(ctx, scoring):
    A, B = synth.random_pair(17, 700, 650, plant_len=300, s=0.1, g=0.02)
    check_stage1(ctx, A, B, scoring, 1)


@pytest.mark.parametrize("delta", [-1, 0, 1])
def test_band_edges(ctx, delta):
    """m around multiples of the band height and of the strip height alpha."""
    g = ctx.row_granularity()
    for bh in (g, g * 32, g * 32 * 4, g * 32 * 8):
        m = bh + delta
        A, B = synth.random_pair(bh + delta + 5, m, 301, plant_len=150)
        check_stage1(ctx, A, B, PAPER, 7)


@pytest.mark.parametrize("k", [2, 3, 7, 16, 32, 100, 512, 2048])
def test_special_row_intervals(ctx, k):
    A, B = synth.random_pair(1000 + k, 4100, 1500, plant_len=1200, s=0.08)
    check_stage1(ctx, A, B, PAPER, k)


def test_ragged_many_tiles(ctx):
    A, B = synth.random_pair(5, 9000, 5003, plant_len=4000, s=0.05, g=0.01)
    check_stage1(ctx, A, B, PAPER, 16)
    check_stage1(ctx, A, B, (2, -1, 4, 1), 0)


def test_ties_low_complexity(ctx):
    # many equal maxima: tie-break (max, min i, min j) (reading S4)
    check_stage1(ctx, "A" * 300, "A" * 200, PAPER, 1)
    check_stage1(ctx, "AC" * 150, "CA" * 170, PAPER, 3)
    check_stage1(ctx, "ACGT" * 600, "ACGT" * 500, PAPER, 64)
    X = synth.random_pair(3, 400, 1)[0]
    XX = np.concatenate([X, X, X])
    check_stage1(ctx, XX, X, PAPER, 1)  # three equal copies: the first wins
    check_stage1(ctx, X, XX, PAPER, 1)


def test_closed_forms(ctx):
    X = synth.random_pair(9, 5000, 1)[0]
    r, _ = ctx.align_stage1(X, X, *PAPER)
    assert r.astuple() == (5000, 5000, 5000)
    r, _ = ctx.align_stage1("AAAAAAAA", "CCCCCCCC", *PAPER)
    assert r.astuple() == (0, 0, 0)
    r, _ = ctx.align_stage1("", "ACGT", *PAPER)
    assert r.astuple() == (0, 0, 0)
    r, rows = ctx.align_stage1("ACGT", "", *PAPER, k=1, keep_rows=True)
    assert r.astuple() == (0, 0, 0) and rows == []


def test_case_insensitive_and_alphabet(ctx):
    from paper_conf_ipps_sandesm11_b200 import SW_EALPHABET, SwError

    A, B = synth.random_pair(12, 900, 800, lower_frac=0.3, plant_len=300)
    check_stage1(ctx, A, B, PAPER, 5)
    with pytest.raises(SwError) as e:
        ctx.align_stage1("ACGTN", "ACGT", *PAPER)
    assert e.value.code == SW_EALPHABET
    with pytest.raises(SwError) as e:
        ctx.align_stage1("ACGT" * 100, "AC-T" * 100, *PAPER, k=4, keep_rows=True)
    assert e.value.code == SW_EALPHABET


def test_bad_parameters(ctx):
    from paper_conf_ipps_sandesm11_b200 import SW_EINVAL, SW_ERANGE, SwError

    for args in [(1, -3, -1, 2), (1, -3, 3, -2)]:  # (200, -3, 3, 2) runs: tests/test_gpu_wide.py
        with pytest.raises(SwError) as e:
            ctx.align_stage1("ACGT", "ACGT", *args)
        assert e.value.code == SW_EINVAL
    with pytest.raises(SwError) as e:
        ctx.align_stage1("ACGT" * 1000, "ACGT" * 1000, 1, -3, 3, 2, k=-1)
    assert e.value.code == SW_EINVAL
    # 2^30 / 100 = 10.7M: a 11M x 11M problem at match 100 could overflow
    import ctypes

    big = 11_000_000
    from paper_conf_ipps_sandesm11_b200 import SINK, _Result

    out = _Result()
    rc = ctx._lib.sw_align_stage1(ctx._h, 1, big, 1, big, 100, -3, 3, 2, 0, SINK(), None, ctypes.byref(out))
    assert rc == SW_ERANGE


@pytest.mark.parametrize("packed", [True, False])
def test_special_rows_streamed_in_chunks(ctx, packed):
    # rows wider than the host's copy chunk (65536 columns): the host copies
    # each row's final columns while its band still runs, then the rest
    A, B = synth.random_pair(77, 8292, 200_003, plant_len=6000, s=0.05, g=0.01)
    ctx.set_kernel(-1, packed)
    try:
        check_stage1(ctx, A, B, PAPER, 2048)
    finally:
        ctx.set_kernel(-1, True)


def test_sink_abort(ctx):
    from paper_conf_ipps_sandesm11_b200 import SW_EABORTED, SwError

    A, B = synth.random_pair(2, 3000, 500)
    seen = []

    def sink(row, H, F):
        seen.append(row)
        return row >= 200

    with pytest.raises(SwError) as e:
        ctx.align_stage1(A, B, *PAPER, k=100, sink=sink)
    assert e.value.code == SW_EABORTED
    assert seen == [100, 200]
    # the context stays usable
    check_stage1(ctx, A, B, PAPER, 100)


def test_repeated_calls_reuse_buffers(ctx):
    for seed, (m, n) in enumerate([(5000, 300), (300, 5000), (2500, 2500), (40, 40)]):
        A, B = synth.random_pair(seed, m, n, plant_len=min(m, n) // 2)
        check_stage1(ctx, A, B, PAPER, 64)


# ---------------------------------------------------------------- reverse pass

def test_reverse_goal_small(ctx):
    done = 0
    for seed in range(40):
        m, n = 50 + 37 * seed, 60 + 29 * seed
        A, B = synth.random_pair(seed, m, n, plant_len=min(m, n) // 2, s=0.08, g=0.02)
        for scoring in (PAPER, (2, -1, 4, 1), (1, -1, 0, 2)):
            (s, ie, je), _ = oracle.stage1(_s(A), _s(B), *scoring)
            if s == 0:
                continue
            want = oracle.reverse_goal(_s(A), ie, _s(B), je, *scoring, s)
            got = ctx.reverse_goal(A, ie, B, je, s, *scoring)
            assert got.astuple() == want, (seed, scoring)
            done += 1
    assert done > 80


def test_reverse_goal_edges(ctx):
    from paper_conf_ipps_sandesm11_b200 import SW_ENOTFOUND, SwError

    assert ctx.reverse_goal("ACGT", 2, "ACGT", 3, 0, *PAPER).astuple() == (0, 2, 3)
    with pytest.raises(SwError) as e:
        ctx.reverse_goal("ACGTACGT", 8, "ACGTACGT", 8, 9, *PAPER)
    assert e.value.code == SW_ENOTFOUND
    X = synth.random_pair(4, 3000, 1)[0]
    assert ctx.reverse_goal(X, 3000, X, 3000, 3000, *PAPER).astuple() == (3000, 0, 0)
    # the Figure-1 pair: two starts tie, the rule picks (2,2) (reading S10)
    assert ctx.reverse_goal("ACTTCCAGA", 9, "AGTTCCGGAGG", 9, 5, 1, -1, 0, 2).astuple() == (5, 2, 2)


def test_reverse_goal_long_alignment(ctx):
    """A whole-length homology: the reverse pass must grow its rectangle to the full matrix."""
    A, B = synth.random_pair(77, 6000, 6000, plant_len=6000, s=0.03, g=0.005)
    (s, ie, je), _ = oracle.stage1(_s(A), _s(B), *PAPER)
    want = oracle.reverse_goal(_s(A), ie, _s(B), je, *PAPER, s)
    got = ctx.reverse_goal(A, ie, B, je, s, *PAPER)
    assert got.astuple() == want


# ---------------------------------------------------------------- the paper-shaped configs

def test_config_c1_full(ctx):
    """BASELINE configs[0]: 50 KBP x 50 KBP with a planted 2 KBP region, k = 1024:
    score, end cell, all 48 special rows and the start cell, bit-exact."""
    cfg = synth.CONFIGS["C1"]
    A, B = synth.make_pair(cfg)
    got = check_stage1(ctx, A, B, PAPER, cfg.k)
    assert got.score > 100  # the plant dominates the background
    want = oracle.reverse_goal(_s(A), got.i, _s(B), got.j, *PAPER, got.score)
    assert ctx.reverse_goal(A, got.i, B, got.j, got.score, *PAPER).astuple() == want
