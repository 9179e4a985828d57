"""Pins for the oracle's Stages 3-5: the alignment of one
partition with crosspoint types and the full optimal local
alignment with its GAP_1 / GAP_2 lists.  Every pin is fixed by
something other than the oracle's own DP: brute-force enumeration of all
alignments, the printed Figure 1 alignment, an independent column scorer
(oracle.brute.score_alignment, itself pinned by Figure 1 and Table X), and
closed forms."""
import itertools
import random

import numpy as np
import pytest

import oracle
from oracle import brute

PAPER = (1, -3, 3, 2)
SCORINGS = [PAPER, (1, -1, 0, 2), (2, -1, 4, 1), (3, -2, 1, 1), (1, -2, 2, 0)]


def _rand(rng, n):
    return "".join(rng.choice("ACGT") for _ in range(n))


def printed(A, B, i0, j0, moves):
    """The alignment as two printed rows ('-' for gaps)."""
    top, bot = [], []
    i, j = i0, j0
    for c in moves:
        if c == "M":
            top.append(A[i]); bot.append(B[j]); i += 1; j += 1
        elif c == "I":
            top.append("-"); bot.append(B[j]); j += 1
        else:
            top.append(A[i]); bot.append("-"); i += 1
    return "".join(top), "".join(bot), i, j


def test_fig1_global_partition_is_printed_alignment_score():
    # Figure 1: the printed alignment scores 1 and is optimal
    g = {}
    for ln in open(__file__.rsplit("/", 1)[0] + "/golden/fig1.txt"):
        if ln.startswith("#") or not ln.strip():
            continue
        key, val = ln.split(None, 1)
        g[key] = val.strip()
    A, B = g["top"].replace("-", ""), g["bottom"].replace("-", "")
    sc = (int(g["match"]), int(g["mismatch"]), int(g["gap_open"]), int(g["gap_ext"]))
    s, mv = oracle.align_partition(A, B, *sc, (0, 0, 0), (len(A), len(B), 0))
    assert s == int(g["score"]) == 1
    top, bot, i, j = printed(A, B, 0, 0, mv)
    assert (i, j) == (len(A), len(B))
    assert brute.score_alignment(top, bot, *sc) == 1


@pytest.mark.parametrize("scoring", SCORINGS)
def test_partition_types_equal_brute_force(scoring):
    rng = random.Random(hash(scoring) & 0xffff)
    for _ in range(25):
        A, B = _rand(rng, rng.randint(0, 5)), _rand(rng, rng.randint(0, 5))
        off_a, off_b = _rand(rng, rng.randint(0, 3)), _rand(rng, rng.randint(0, 3))
        SA, SB = off_a + A + _rand(rng, 2), off_b + B + _rand(rng, 2)
        for ts, te in itertools.product(range(3), range(3)):
            want = brute.partition_best(A, B, *scoring, ts, te)
            Cs = (len(off_a), len(off_b), ts)
            Ce = (len(off_a) + len(A), len(off_b) + len(B), te)
            got, mv = oracle.align_partition(SA, SB, *scoring, Cs, Ce)
            assert got == want, (A, B, scoring, ts, te)
            if got is None:
                continue
            # the moves consume the partition exactly and rescore to the optimum:
            # a gap run that continues the start state is charged without an opening
            top, bot, i, j = printed(SA, SB, Cs[0], Cs[1], mv)
            assert (i, j) == Ce[:2]
            go, ge = scoring[2], scoring[3]
            refund = 0
            if ts == 1 and mv.startswith("I"):
                refund = go
            if ts == 2 and mv.startswith("D"):
                refund = go
            assert brute.score_alignment(top, bot, *scoring) + refund == got
            if not mv:
                assert te in (0, ts)  # the empty alignment stays in the start state
            elif te == 1:
                assert mv.endswith("I")
            elif te == 2:
                assert mv.endswith("D")


def test_global_partition_equals_global_score():
    rng = random.Random(5)
    for _ in range(40):
        A, B = _rand(rng, rng.randint(1, 40)), _rand(rng, rng.randint(1, 40))
        for sc in SCORINGS:
            s, _ = oracle.align_partition(A, B, *sc, (0, 0, 0), (len(A), len(B), 0))
            assert s == oracle.global_score(A, B, *sc)


def _check_alignment(A, B, sc, r):
    top, bot, i, j = printed(A, B, r["start"][0], r["start"][1], r["moves"])
    assert (i, j) == r["end"]
    assert brute.score_alignment(top, bot, *sc) == r["score"]
    # GAP lists re-derive the move string
    i, j = r["start"]
    events = sorted([(gi, gj, L, "I") for gi, gj, L in r["gap1"]] + [(gi, gj, L, "D") for gi, gj, L in r["gap2"]])
    mv = []
    for gi, gj, L, c in events:
        d = gi - i
        assert d >= 0 and gj - j == d, "pairs between gap runs run diagonally"
        mv.append("M" * d)
        mv.append(c * L)
        i, j = (gi, gj + L) if c == "I" else (gi + L, gj)
    d = r["end"][0] - i
    assert d >= 0 and r["end"][1] - j == d
    mv.append("M" * d)
    assert "".join(mv) == r["moves"]


@pytest.mark.parametrize("scoring", SCORINGS)
def test_full_alignment_brute_force_tiny(scoring):
    rng = random.Random(7 + hash(scoring) % 100)
    for _ in range(30):
        A, B = _rand(rng, rng.randint(1, 6)), _rand(rng, rng.randint(1, 6))
        best = brute.local_best(A, B, *scoring)
        for k in (0, 1, 2, 3):
            r = oracle.align(A, B, *scoring, k)
            assert r["score"] == best[0]
            assert r["end"] == ((best[1], best[2]) if best[0] > 0 else (0, 0))
            if best[0] > 0:
                _check_alignment(A, B, scoring, r)


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_full_alignment_planted_medium(seed):
    import synth

    A, B = synth.random_pair(seed, 900, 800, plant_len=500, s=0.05, g=0.01)
    A, B = A.tobytes().decode(), B.tobytes().decode()
    for sc in SCORINGS[:3]:
        (best, ie, je), _ = oracle.stage1(A, B, *sc, k=0, keep_rows=False)
        for k in (16, 100, 1000):
            r = oracle.align(A, B, *sc, k)
            assert r["score"] == best and r["end"] == (ie, je)
            _check_alignment(A, B, sc, r)
            assert r["crosspoints"][0][:2] == r["start"]


def test_closed_forms():
    rng = random.Random(11)
    X = _rand(rng, 60)
    r = oracle.align(X, X, *PAPER, 16)
    assert r["moves"] == "M" * 60 and r["start"] == (0, 0) and r["gap1"] == r["gap2"] == []
    # one inserted run of 5 in the middle: 60 matches - (3 + 2*5) beats either half alone
    Y = X[:30] + "TTTTT" + X[30:]
    r = oracle.align(X, Y, *PAPER, 16)
    assert r["score"] == 60 - (3 + 2 * 5)
    assert r["gap2"] == [] and len(r["gap1"]) == 1 and r["gap1"][0][2] == 5
    _check_alignment(X, Y, PAPER, r)
    r = oracle.align(Y, X, *PAPER, 7)
    assert r["gap1"] == [] and len(r["gap2"]) == 1 and r["gap2"][0][2] == 5
    _check_alignment(Y, X, PAPER, r)
