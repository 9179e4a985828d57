"""Stage 2 (N1) on the GPU against the oracle: the crosspoint list L_2 must be
identical (every crosspoint's i, j, score and type, in order).  Covers gap
crosspoints (F junctions), several scorings and special-row intervals, ties
on low-complexity input, partitions wider than one band of the transposed
fill (so the first-event abort runs), the int32 kernel geometries, and C1
end to end.  Also: the start point agrees with the reverse pass where the
optimal alignment is unique, and the preconditions are enforced."""
import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu
PAPER = (1, -3, 3, 2)
SCORINGS = [PAPER, (2, -1, 4, 1), (1, -1, 0, 2), (5, -4, 10, 1), (3, -2, 0, 1)]


@pytest.fixture(scope="module")
def ctx():
    from paper_conf_ipps_sandesm11_b200 import Context, build

    build.build()
    c = Context(0)
    yield c
    c.set_kernel(-1, True)
    c.close()


def _s(x):
    return x.tobytes().decode() if isinstance(x, np.ndarray) else x


def check(ctx, A, B, sc, k):
    got1, _ = ctx.align_stage1(A, B, *sc, k=k)
    (best, ie, je), _ = oracle.stage1(_s(A), _s(B), *sc, k=0)
    assert got1.astuple() == (best, ie, je)
    L = ctx.stage2(A, B, *sc, k=k, end=got1)
    want = oracle.stage2(_s(A), _s(B), *sc, k, best, ie, je)
    assert L == want, (len(A), len(B), sc, k)
    return L


def test_planted_gap_crosspoints(ctx):
    X = "ACGTTGCAACGGTACCTGAT"
    Y = "GGCATTACGATCCAGTACGA"
    A, B = X + "TTTT" + Y, X + Y
    assert check(ctx, A, B, PAPER, 22) == [(0, 0, 0, 0), (22, 20, 13, 2), (44, 40, 29, 0)]
    L = check(ctx, A, B, PAPER, 1)
    assert L[21:25] == [(21, 20, 15, 2), (22, 20, 13, 2), (23, 20, 11, 2), (24, 20, 9, 0)]
    # the same gap in the other sequence: a horizontal gap crossing no special row
    check(ctx, B, A, PAPER, 7)


@pytest.mark.parametrize("seed", range(5))
def test_random_small(ctx, seed):
    sc = SCORINGS[seed]
    A, B = synth.random_pair(300 + seed, 160 + 7 * seed, 150, plant_len=120, s=0.08, g=0.04, mu=3)
    for k in (1, 3, 16, 40, 500, 0):
        check(ctx, A, B, sc, k)


@pytest.mark.parametrize("k", [16, 64, 257, 1024])
def test_gapped_medium(ctx, k):
    # partitions up to 1024 rows, S1 prefixes longer than one 4096-row band of
    # the transposed fill: bands after the first event abort
    A, B = synth.random_pair(41 + k, 6000, 9500, plant_len=5000, s=0.04, g=0.006, mu=4)
    check(ctx, A, B, PAPER, k)


def test_scorings_medium(ctx):
    A, B = synth.random_pair(77, 3000, 5200, plant_len=2500, s=0.05, g=0.01, mu=3)
    for sc in SCORINGS:
        check(ctx, A, B, sc, 128)


def test_ties_low_complexity(ctx):
    X = synth.random_pair(3, 300, 1)[0]
    XXX = np.concatenate([X, X, X])
    for k in (50, 64, 300):
        check(ctx, XXX, X, PAPER, k)
        check(ctx, X, XXX, PAPER, k)
    rep = np.frombuffer(b"ACACACACAC" * 60, dtype=np.uint8)
    rep2 = np.frombuffer(b"ACACACAAC" * 61, dtype=np.uint8)
    check(ctx, rep, rep2, PAPER, 37)
    check(ctx, rep, rep2, (1, -1, 0, 2), 16)


@pytest.mark.parametrize("variant", [0, 2, 7])
def test_int32_geometries(ctx, variant):
    A, B = synth.random_pair(500 + variant, 4000, 6000, plant_len=3500, s=0.04, g=0.01, mu=3)
    ctx.set_kernel(variant, False)
    try:
        check(ctx, A, B, PAPER, 256)
    finally:
        ctx.set_kernel(-1, True)


def test_start_matches_reverse_pass_when_unique(ctx):
    # a gapless plant in random background: one optimal alignment
    A, B = synth.random_pair(9, 20000, 15000, plant_len=900, s=0.02, g=0.0)
    r, _ = ctx.align_stage1(A, B, *PAPER, k=256)
    L = ctx.stage2(A, B, *PAPER, k=256, end=r)
    st = ctx.reverse_goal(A, r.i, B, r.j, r.score, *PAPER)
    assert L[0][:2] == (st.i, st.j)
    assert L[-1] == (r.i, r.j, r.score, 0)


def test_config_c1(ctx):
    cfg = synth.CONFIGS["C1"]
    A, B = synth.make_pair(cfg)
    L = check(ctx, A, B, PAPER, cfg.k)
    assert len(L) >= 2


def test_preconditions(ctx):
    from paper_conf_ipps_sandesm11_b200 import SW_EINVAL, SwError

    A, B = synth.random_pair(1, 2000, 1800, plant_len=1000)
    r, _ = ctx.align_stage1(A, B, *PAPER, k=64)
    with pytest.raises(SwError) as e:
        ctx.stage2(A, B, *PAPER, k=32, end=r)  # rows of another interval
    assert e.value.code == SW_EINVAL
    with pytest.raises(SwError) as e:
        ctx.stage2(A, B, 2, -1, 4, 1, k=64, end=r)  # another scoring
    assert e.value.code == SW_EINVAL
    ctx.reverse_goal(A, r.i, B, r.j, r.score, *PAPER)  # a reverse pass keeps the rows
    assert ctx.stage2(A, B, *PAPER, k=64, end=r)[-1] == (r.i, r.j, r.score, 0)
    ctx.set_virtual_stripes(2)
    try:
        r2, _ = ctx.align_stage1(A, B, *PAPER, k=64)
    finally:
        ctx.set_virtual_stripes(1)
    with pytest.raises(SwError) as e:
        ctx.stage2(A, B, *PAPER, k=64, end=r2)  # rows split over virtual stripes
    assert e.value.code == SW_EINVAL
    # best score 0: the list is the start point alone
    r0, _ = ctx.align_stage1("AAAA", "CCCC", *PAPER, k=2)
    assert r0.astuple() == (0, 0, 0)
    assert ctx.stage2("AAAA", "CCCC", *PAPER, k=2, end=r0) == [(0, 0, 0, 0)]
