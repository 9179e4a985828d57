"""The reverse pass (a8) on the packed 16x2 kernel in global mode (DESIGN.md
4.6): the start cell is identical to the oracle's and to the int32 kernel's
on random, gapped, whole-length, tie-prone and edge inputs, and the packed
(immediate-patched) kernel is the one that ran."""
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
    c.set_kernel(-1, True)
    c.close()


def _s(x):
    return x.tobytes().decode() if isinstance(x, np.ndarray) else x


def both(ctx, A, ie, B, je, goal, scoring):
    ctx.set_kernel(-1, True)
    p = ctx.reverse_goal(A, ie, B, je, goal, *scoring).astuple()
    st = ctx.stats()
    ctx.set_kernel(1, False)  # int32 kernel, default geometry
    try:
        q = ctx.reverse_goal(A, ie, B, je, goal, *scoring).astuple()
        st2 = ctx.stats()
    finally:
        ctx.set_kernel(-1, True)
    assert st2["alpha"] > 0, st2
    return p, q, st


@pytest.mark.parametrize("scoring", [PAPER, (2, -1, 4, 1), (1, -1, 0, 2), (3, -2, 2, 3)])
def test_reverse_packed_random(ctx, scoring):
    done = 0
    for seed in range(24):
        m, n = 300 + 411 * seed, 280 + 397 * seed
        A, B = synth.random_pair(100 + seed, m, n, plant_len=min(m, n) // 2, s=0.06, g=0.02)
        (s, ie, je), _ = oracle.stage1(_s(A), _s(B), *scoring)
        if s == 0:
            continue
        want = oracle.reverse_goal(_s(A), ie, _s(B), je, *scoring, s)
        p, q, st = both(ctx, A, ie, B, je, s, scoring)
        assert p == want and q == want, (seed, scoring, p, q, want)
        assert st["alpha"] < 0 and st["patched"] == 1, st
        done += 1
    assert done >= 20


def test_reverse_packed_whole_length(ctx):
    """Whole-length homology: the reverse pass covers (nearly) the full matrix,
    several bands and tiles of the packed geometry (8192-row bands)."""
    for seed, L in ((7, 9000), (8, 17000)):
        A, B = synth.random_pair(seed, L, L, plant_len=L, s=0.02, g=0.004)
        (s, ie, je), _ = oracle.stage1(_s(A), _s(B), *PAPER)
        want = oracle.reverse_goal(_s(A), ie, _s(B), je, *PAPER, s)
        p, q, st = both(ctx, A, ie, B, je, s, PAPER)
        assert p == want and q == want, (seed, p, q, want)
        assert st["alpha"] < 0


def test_reverse_packed_ties_and_edges(ctx):
    # low-complexity sequences: many cells equal the goal, the first one in row-major order wins
    rng = np.random.default_rng(5)
    for trial in range(6):
        A = np.frombuffer(("AC" * 1500).encode(), dtype=np.uint8).copy()
        B = np.frombuffer(("AC" * 1400 + "GT" * 50).encode(), dtype=np.uint8).copy()
        A[rng.integers(0, len(A), 20)] = ord("G")
        (s, ie, je), _ = oracle.stage1(_s(A), _s(B), *PAPER)
        want = oracle.reverse_goal(_s(A), ie, _s(B), je, *PAPER, s)
        p, q, st = both(ctx, A, ie, B, je, s, PAPER)
        assert p == want and q == want, (trial, p, q, want)
    # the Figure-1 pair (reading S10: starts (2,2) and (0,0) tie, (2,2) wins)
    p, q, _ = both(ctx, "ACTTCCAGA", 9, "AGTTCCGGAGG", 9, 5, (1, -1, 0, 2))
    assert p == q == (5, 2, 2)
    X = synth.random_pair(4, 3000, 1)[0]
    p, q, _ = both(ctx, X, 3000, X, 3000, 3000, PAPER)
    assert p == q == (3000, 0, 0)


@pytest.mark.parametrize("scoring", [(5, -4, 10, 5), (1, -1, 0, 1), (4, -5, 0, 7)])
def test_reverse_packed_window_edges(ctx, scoring):
    """Scorings near the packed kernel's 16-bit window bound (DESIGN.md 4.7:
    (32 alpha + 140)(|p|max + G_first) + 1024 < 30000) and the smallest
    penalties, on a whole-length pair: Stage 1 and the reverse pass both
    packed, bit-exact."""
    A, B = synth.random_pair(31 + scoring[2], 6000, 5800, plant_len=6000, s=0.03, g=0.006)
    got, _ = ctx.align_stage1(A, B, *scoring, k=0)
    assert ctx.stats()["alpha"] < 0
    (s, ie, je), _ = oracle.stage1(_s(A), _s(B), *scoring)
    assert got.astuple() == (s, ie, je)
    want = oracle.reverse_goal(_s(A), ie, _s(B), je, *scoring, s)
    p, q, st = both(ctx, A, ie, B, je, s, scoring)
    assert p == want and q == want, (scoring, p, q, want)
    assert st["alpha"] < 0
