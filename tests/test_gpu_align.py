"""Stages 3-5 on the GPU (sw_align: Myers-Miller with balanced splitting, then
full traceback of small partitions) against the oracle's full
alignment (oracle.align).  Several alignments can be optimal, so the test
compares what is unique -- score, start point, end point -- and checks that
the GPU alignment is valid: its GAP_1 / GAP_2 lists rebuild a path from
the start to the end point that the independent column scorer rescores to the
optimal score."""
import numpy as np
import pytest

import oracle
import synth
from oracle import brute

pytestmark = pytest.mark.gpu
PAPER = (1, -3, 3, 2)
SCORINGS = [PAPER, (1, -1, 0, 2), (2, -1, 4, 1), (5, -4, 10, 1), (1, -2, 2, 0)]


@pytest.fixture(scope="module")
def ctx():
    from paper_conf_ipps_sandesm11_b200 import Context, build

    build.build()
    c = Context(0)
    yield c
    c.close()


def _s(x):
    return x.tobytes().decode() if isinstance(x, np.ndarray) else x


def rebuild(r):
    """Move string from the GAP lists: pairs run diagonally between gap runs."""
    (i, j), mv = r["start"], []
    ev = sorted([(gi, gj, L, "I") for gi, gj, L in r["gap1"]] + [(gi, gj, L, "D") for gi, gj, L in r["gap2"]])
    for gi, gj, L, c in ev:
        d = gi - i
        assert d >= 0 and gj - j == d, (gi, gj, i, j)
        mv.append("M" * d + c * L)
        i, j = (gi, gj + L) if c == "I" else (gi + L, gj)
    d = r["end"][0] - i
    assert d >= 0 and r["end"][1] - j == d
    mv.append("M" * d)
    return "".join(mv)


def rescore(A, B, r, sc):
    top, bot = [], []
    i, j = r["start"]
    for c in rebuild(r):
        if c == "M":
            top.append(A[i]); bot.append(B[j]); i += 1; j += 1
        elif c == "I":
            top.append("-"); bot.append(B[j]); j += 1
        else:
            top.append(A[i]); bot.append("-"); i += 1
    assert (i, j) == r["end"]
    return brute.score_alignment("".join(top), "".join(bot), *sc)


def check(ctx, A, B, sc, k, want_levels=None):
    A, B = _s(A), _s(B)
    got = ctx.align(A, B, *sc, k=k)
    want = oracle.align(A, B, *sc, k)
    assert (got["score"], got["start"], got["end"]) == (want["score"], want["start"], want["end"]), (sc, k)
    if got["score"] > 0:
        assert rescore(A, B, got, sc) == got["score"]
    if want_levels is not None:
        assert got["mm_levels"] >= want_levels, got
    return got


@pytest.mark.parametrize("sc", SCORINGS)
def test_align_small_random(ctx, sc):
    for seed in range(4):
        A, B = synth.random_pair(300 + seed, 700 + 50 * seed, 600, plant_len=400, s=0.06, g=0.02)
        for k in (0, 16, 64, 128):
            check(ctx, A, B, sc, k)


def test_align_tiny_and_degenerate(ctx):
    check(ctx, "A", "A", PAPER, 0)
    check(ctx, "A", "C", PAPER, 0)
    check(ctx, "ACGT", "TTTT", PAPER, 16)
    X = _s(synth.random_pair(9, 200, 1)[0])
    r = check(ctx, X, X, PAPER, 16)
    assert r["gap1"] == r["gap2"] == [] and r["start"] == (0, 0)
    Y = X[:100] + "GGGGG" + X[100:]
    r = check(ctx, X, Y, PAPER, 32)
    assert r["gap2"] == [] and [g[2] for g in r["gap1"]] == [5]
    r = check(ctx, Y, X, PAPER, 32)
    assert r["gap1"] == [] and [g[2] for g in r["gap2"]] == [5]


@pytest.mark.parametrize("sc", [PAPER, (2, -1, 4, 1), (1, -1, 0, 2)])
def test_align_forces_myers_miller_splits(ctx, sc):
    # whole-length homology, one Stage-2 partition (k = 0) of ~9e6 cells: several split levels,
    # split in rows and (for the wide pair) in columns, gap crosspoints included
    A, B = synth.random_pair(77, 3000, 3000, plant_len=3000, s=0.03, g=0.01)
    check(ctx, A, B, sc, 0, want_levels=3)
    A, B = synth.random_pair(78, 600, 4000, plant_len=600, s=0.03, g=0.02)
    check(ctx, A, B, sc, 0, want_levels=2)
    check(ctx, B, A, sc, 256, want_levels=1)


def test_align_cta_split_many_chunks(ctx):
    # 12000-row partitions: the CTA split kernel runs 6000-row passes as 24 chunks on 8 warps
    # (ring slots reused), in rows and -- for the transposed pair -- in columns
    A, B = synth.random_pair(91, 12000, 3000, plant_len=3000, s=0.02, g=0.01)
    A = A[:]
    check(ctx, A, B, PAPER, 0, want_levels=3)
    check(ctx, B, A, (2, -1, 4, 1), 0, want_levels=3)


def test_align_long_gaps(ctx):
    rng = np.random.default_rng(5)
    X = "".join(rng.choice(list("ACGT"), 2500))
    Y = X[:800] + "".join(rng.choice(list("ACGT"), 300)) + X[800:1700] + X[1900:]
    for sc in (PAPER, (2, -1, 4, 1)):
        for k in (0, 64, 512):
            check(ctx, X, Y, sc, k)
            check(ctx, Y, X, sc, k)


def test_align_config_c1(ctx):
    cfg = synth.CONFIGS["C1"]
    A, B = synth.make_pair(cfg)
    r = check(ctx, A, B, PAPER, cfg.k)
    assert r["partitions"] >= 1
