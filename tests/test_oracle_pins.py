"""Pins for the CPU oracle (oracle/) against things other than itself:
values the paper prints, brute-force enumeration of alignments, closed forms,
an independent textbook recurrence, and invariants.
No GPU needed."""
import itertools
import os
import random

import numpy as np
import pytest

import oracle
from oracle import brute
import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden")
PAPER = (1, -3, 3, 2)  # P:315 via reading S2: match +1, mismatch -3, G_open 3, G_ext 2


def _read_golden(name):
    out = {}
    with open(os.path.join(GOLD, name)) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            k, *v = line.split()
            out[k] = v
    return out


def _rand_seq(rng, n):
    return "".join(rng.choice("ACGT") for _ in range(n))


# ---------------------------------------------------------------- Figure 1

def test_fig1_rescore_printed_alignment():
    g = _read_golden("fig1.txt")
    top, bottom = g["top"][0], g["bottom"][0]
    ma, mi, go, ge = (int(g[k][0]) for k in ("match", "mismatch", "gap_open", "gap_ext"))
    cols = [int(x) for x in g["columns"]]
    # column by column
    assert len(cols) == len(top) == len(bottom) == 11
    assert sum(cols) == int(g["score"][0]) == 1
    assert brute.score_alignment(top, bottom, ma, mi, go, ge) == 1


def test_fig1_global_optimum_is_printed_score():
    """The printed Figure-1 alignment is optimal: the NW optimum of S0 vs S1 under
    the figure's scoring equals the printed score 1 -- by explicit enumeration
    (brute) and by the oracle's global recurrence."""
    g = _read_golden("fig1.txt")
    S0 = g["top"][0].replace("-", "")
    S1 = g["bottom"][0].replace("-", "")
    assert (S0, S1) == ("ACTTCCAGA", "AGTTCCGGAGG")
    args = (1, -1, 0, 2)
    assert brute.global_best(S0, S1, *args) == 1
    assert oracle.global_score(S0, S1, *args) == 1


def test_fig1_local_regression_values():
    """Derived (unprinted) values on the Figure-1 pair, fixed as regressions
    (SURVEY.md 8(c)): (+1,-1,0,2) best 5 at (9,9); paper scoring best 4 at
    (6,6) and NW -6.  Checked by the full-matrix and linear-space variants."""
    S0, S1 = "ACTTCCAGA", "AGTTCCGGAGG"
    (s, i, j), _ = oracle.stage1(S0, S1, 1, -1, 0, 2)
    assert (s, i, j) == (5, 9, 9)
    H, _, _ = oracle.full_matrix(S0, S1, 1, -1, 0, 2)
    assert H.max() == 5 and int((H == 5).sum()) == 1 and H[9, 9] == 5
    (s, i, j), _ = oracle.stage1(S0, S1, *PAPER)
    assert (s, i, j) == (4, 6, 6)
    assert oracle.global_score(S0, S1, *PAPER) == -6
    assert brute.global_best(S0, S1, *PAPER) == -6
    # reverse pass tie (reading S10): starts (2,2) and (0,0) both score 5; the rule picks (2,2)
    starts = brute.all_local_starts(S0, S1, 1, -1, 0, 2, 9, 9, 5)
    assert starts == {(2, 2), (0, 0)}
    assert oracle.reverse_goal(S0, 9, S1, 9, 1, -1, 0, 2, 5) == (5, 2, 2)


# ---------------------------------------------------------------- Table X / III

def test_table_x_cost_model():
    """Affine cost model: a run of L gap columns costs G_first + (L-1) G_ext with
    G_first = 5, G_ext = 2; with the API's gap_open = G_first - G_ext = 3
     the printed composition reproduces the printed score exactly."""
    g = _read_golden("table_x.txt")
    ma, mi, go, ge = PAPER
    nm, sm = (int(x) for x in g["matches"])
    nx, sx = (int(x) for x in g["mismatches"])
    no, so = (int(x) for x in g["gap_openings"])
    ne, se = (int(x) for x in g["gap_extensions"])
    tot, stot = (int(x) for x in g["total"])
    assert sm == nm * ma and sx == nx * mi
    assert so == -no * (go + ge)  # each opening column costs G_first = 5
    assert se == -ne * ge
    assert sm + sx + so + se == stot == 27206434
    assert nm + nx + no + ne == tot  # columns = alignment length (Table III)
    assert no + ne == int(g["table3_gaps"][0])
    # the competing reading (gap_open = G_first, a run costs 5 + 2L) does not fit
    assert nm * ma + nx * mi - no * (5 + 2) - ne * 2 != stot


def test_table_x_composition_rescores_via_alignment_scorer():
    """A literal alignment with Table X's proportions (scaled down) rescored
    column by column equals the closed form used above."""
    top = "ACGT" * 5 + "A" * 3 + "--" + "TTT" + "-" * 5 + "G"
    bot = "ACGT" * 5 + "ACC" + "GG" + "TTT" + "CCCCC" + "G"
    ma, mi, go, ge = PAPER
    # 20 + 3 + 3 + 1 = 27 pair columns, 2 mismatches (A/C, A/C); two gap runs (2 and 5)
    matches = sum(1 for a, b in zip(top, bot) if a != "-" and b != "-" and a == b)
    mism = sum(1 for a, b in zip(top, bot) if a != "-" and b != "-" and a != b)
    expect = matches * ma + mism * mi - (go + ge) * 2 - ge * (1 + 4)
    assert brute.score_alignment(top, bot, ma, mi, go, ge) == expect


# ---------------------------------------------------------------- brute force (Eq. 1-3 as a max over alignments)

SCORINGS = [PAPER, (1, -1, 0, 2), (2, -1, 4, 1), (3, -2, 0, 1), (1, -3, 10, 1), (5, -4, 1, 3)]


@pytest.mark.parametrize("scoring", SCORINGS)
def test_full_matrix_equals_brute_force(scoring):
    rng = random.Random(hash(scoring) & 0xFFFF)
    for _ in range(12):
        m, n = rng.randint(0, 5), rng.randint(0, 5)
        A, B = _rand_seq(rng, m), _rand_seq(rng, n)
        Hb, Eb, Fb = brute.local_matrices(A, B, *scoring)
        H, E, F = oracle.full_matrix(A, B, *scoring)
        for i in range(m + 1):
            for j in range(n + 1):
                assert H[i, j] == Hb[i][j], (A, B, i, j)
                if i == 0 or j == 0:
                    continue  # E, F on the boundary are not defined by Eq. 2-3 (reading S3)
                if Eb[i][j] is None:
                    assert E[i, j] <= oracle.NEG // 2
                else:
                    assert E[i, j] == Eb[i][j], (A, B, i, j, "E")
                if Fb[i][j] is None:
                    assert F[i, j] <= oracle.NEG // 2
                else:
                    assert F[i, j] == Fb[i][j], (A, B, i, j, "F")


def test_stage1_best_equals_brute_force_many():
    rng = random.Random(7)
    for t in range(150):
        scoring = SCORINGS[t % len(SCORINGS)]
        m, n = rng.randint(0, 6), rng.randint(0, 6)
        A = _rand_seq(rng, m) if t % 3 else _rand_seq(rng, m).replace("G", "A").replace("T", "C")
        B = _rand_seq(rng, n) if t % 3 else _rand_seq(rng, n).replace("G", "A").replace("T", "C")
        want = brute.local_best(A, B, *scoring)
        got, _ = oracle.stage1(A, B, *scoring)
        assert got == want, (A, B, scoring)


def test_global_equals_brute_force():
    rng = random.Random(11)
    for t in range(60):
        scoring = SCORINGS[t % len(SCORINGS)]
        A, B = _rand_seq(rng, rng.randint(0, 6)), _rand_seq(rng, rng.randint(0, 6))
        assert oracle.global_score(A, B, *scoring) == brute.global_best(A, B, *scoring), (A, B, scoring)


# ---------------------------------------------------------------- textbook special case

def _textbook_linear_sw(A, B, ma, mi, g):
    """Original SW with a linear gap (one matrix): independent recurrence."""
    m, n = len(A), len(B)
    H = [[0] * (n + 1) for _ in range(m + 1)]
    for i in range(1, m + 1):
        for j in range(1, n + 1):
            s = ma if A[i - 1] == B[j - 1] else mi
            H[i][j] = max(0, H[i - 1][j - 1] + s, H[i - 1][j] - g, H[i][j - 1] - g)
    return H


def test_linear_gap_reduces_to_textbook_sw():
    rng = random.Random(5)
    for t in range(25):
        m, n = rng.randint(1, 40), rng.randint(1, 40)
        A, B = _rand_seq(rng, m), _rand_seq(rng, n)
        ma, mi, g = rng.choice([(1, -1, 2), (2, -1, 1), (1, -3, 2), (3, -2, 4)])
        Ht = _textbook_linear_sw(A, B, ma, mi, g)
        H, _, _ = oracle.full_matrix(A, B, ma, mi, 0, g)
        assert (H == np.array(Ht)).all()


# ---------------------------------------------------------------- linear space == full matrix

@pytest.mark.parametrize("k", [1, 2, 3, 7])
def test_linear_space_rows_equal_full_matrix(k):
    rng = random.Random(100 + k)
    for _ in range(6):
        m, n = rng.randint(1, 60), rng.randint(1, 60)
        A, B = _rand_seq(rng, m), _rand_seq(rng, n)
        for scoring in (PAPER, (2, -1, 4, 1)):
            H, E, F = oracle.full_matrix(A, B, *scoring)
            best, rows = oracle.stage1(A, B, *scoring, k=k)
            assert [r for r, _, _ in rows] == list(range(k, m + 1, k))
            for r, h, f in rows:
                assert (h == H[r, 1:]).all() and (f == F[r, 1:]).all()
            # argmax order (max, min i, min j) == first row-major hit (reading S4)
            s = H.max()
            if s == 0:
                assert best == (0, 0, 0)
            else:
                ii, jj = np.argwhere(H == s)[0]
                assert best == (s, ii, jj)


# ---------------------------------------------------------------- closed forms

def test_closed_forms():
    rng = random.Random(3)
    X = _rand_seq(rng, 40)
    assert oracle.stage1(X, X, *PAPER)[0] == (40, 40, 40)
    assert oracle.stage1(X, X, 2, -1, 3, 1)[0] == (80, 40, 40)
    Y = X[:20] + {"A": "C", "C": "G", "G": "T", "T": "A"}[X[20]] + X[21:]
    # one substitution in the middle: 39 matches - 3 = 36 beats either half (<= 20)
    assert oracle.stage1(X, Y, *PAPER)[0] == (36, 40, 40)
    assert oracle.stage1("AAAA", "CCCC", *PAPER)[0] == (0, 0, 0)
    assert oracle.stage1("", "ACGT", *PAPER)[0] == (0, 0, 0)
    assert oracle.stage1("ACGT", "", *PAPER)[0] == (0, 0, 0)
    for L in (1, 2, 5):
        Z = X[:20] + "T" * L + X[20:]
        s = oracle.stage1(X, Z, *PAPER)[0][0]
        assert s >= 40 - (3 + 2 * L)  # one inserted run of length L


def test_case_insensitive():
    rng = random.Random(9)
    A, B = _rand_seq(rng, 50), _rand_seq(rng, 50)
    assert oracle.stage1(A.lower(), B, *PAPER)[0] == oracle.stage1(A, B.lower(), *PAPER)[0] == oracle.stage1(A, B, *PAPER)[0]


# ---------------------------------------------------------------- invariants

COMP = str.maketrans("ACGT", "TGCA")


def test_invariants():
    rng = random.Random(21)
    for t in range(120):
        m, n = rng.randint(1, 45), rng.randint(1, 45)
        A, B = _rand_seq(rng, m), _rand_seq(rng, n)
        scoring = SCORINGS[t % len(SCORINGS)]
        (s, i, j), rows = oracle.stage1(A, B, *scoring, k=1)
        (s2, i2, j2), _ = oracle.stage1(B, A, *scoring)
        assert s == s2 >= 0
        assert s <= min(m, n) * scoring[0]
        # reverse both + complement both
        Ar, Br = A[::-1].translate(COMP), B[::-1].translate(COMP)
        assert oracle.stage1(Ar, Br, *scoring)[0][0] == s
        H, _, _ = oracle.full_matrix(A, B, *scoring)
        if s > 0 and int((H == s).sum()) == 1:
            assert (i2, j2) == (j, i)  # transposes when unique
        gf = scoring[2] + scoring[3]
        for _, h, f in rows:
            assert (f >= -gf).all() and (h >= 0).all()


# ---------------------------------------------------------------- reverse pass

def test_reverse_goal_matches_brute_starts():
    rng = random.Random(31)
    done = 0
    for t in range(400):
        m, n = rng.randint(1, 6), rng.randint(1, 6)
        A, B = _rand_seq(rng, m), _rand_seq(rng, n)
        scoring = SCORINGS[t % len(SCORINGS)]
        (s, ie, je), _ = oracle.stage1(A, B, *scoring)
        if s == 0:
            continue
        starts = brute.all_local_starts(A, B, *scoring, ie, je, s)
        assert starts
        got = oracle.reverse_goal(A, ie, B, je, *scoring, s)
        # first hit in reverse row-major order = largest i_s, then largest j_s (reading S10)
        assert got == (s,) + max(starts), (A, B, scoring)
        done += 1
    assert done > 100


def test_reverse_goal_invariants_medium():
    for seed in range(6):
        A, B = synth.random_pair(seed, 300, 280, plant_len=120)
        A, B = A.tobytes().decode(), B.tobytes().decode()
        for scoring in (PAPER, (2, -1, 4, 1)):
            (s, ie, je), _ = oracle.stage1(A, B, *scoring)
            st = oracle.reverse_goal(A, ie, B, je, *scoring, s)
            assert st is not None and st[0] == s
            _, i_s, j_s = st
            assert 0 <= i_s < ie and 0 <= j_s < je
            # NW of the aligned substrings is the goal; every prefix H <= goal
            assert oracle.global_score(A[i_s:ie], B[j_s:je], *scoring) == s
    assert oracle.reverse_goal("ACGT", 2, "ACGT", 3, *PAPER, 0) == (0, 2, 3)
    assert oracle.reverse_goal("ACGT", 4, "ACGT", 4, *PAPER, 5) is None  # goal > any score


# ---------------------------------------------------------------- band induction

def test_band_induction():
    A, B = synth.random_pair(4, 257, 190, plant_len=90)
    k = 32
    (s, i, j), rows = oracle.stage1(A, B, *PAPER, k=k)
    n = len(B)
    Htop = np.zeros(n + 1, np.int64)
    Ftop = np.full(n + 1, oracle.NEG, np.int64)
    bests = []
    r = 0
    for rr, h, f in rows + [(len(A), None, None)]:
        Hb, Fb, bb = oracle.band(A, B, *PAPER, r, rr, Htop, Ftop)
        if h is not None:
            assert (Hb[1:] == h).all() and (Fb[1:] == f).all()
        bests.append(bb)
        Htop, Ftop, r = Hb, Fb, rr
    top = max(bests, key=lambda x: (x[0], -x[1], -x[2]))
    assert top == (s, i, j)


# ---------------------------------------------------------------- flush-interval rule vs Table VIII

def test_flush_interval_reproduces_table_viii():
    m, n, alphaT, end_row = 32_799_110, 46_944_323, 4 * 64, 32_718_231
    rows = [l.split() for l in open(os.path.join(GOLD, "table_viii.txt")) if l.strip() and not l.startswith("#")]
    for sra_gib, printed in rows:
        R = oracle.flush_rows(m, n, alphaT, int(sra_gib) << 30)
        assert R % alphaT == 0
        predicted = end_row // R + 2  # special rows crossed + start + end point
        if int(sra_gib) in (10, 30, 50):
            assert predicted == int(printed)
        else:
            assert abs(predicted - int(printed)) <= 1
    # SRA of 50 GiB gives R = 229,632 rows
    assert oracle.flush_rows(m, n, alphaT, 50 << 30) == 229_632


# ---------------------------------------------------------------- Stage 2
#
# or_stage2 is pinned by (1) closed forms of a planted gap crossing special
# rows, (2) the partition property S(C_s, C_e) = score_e - score_s
# checked with an independent, test-local Gotoh that honours the crosspoint
# types (a segment leaving a gap crosspoint continues its vertical gap at
# G_ext per row; a segment entering one ends with a vertical gap), (3) the
# start point rescored with the pinned global oracle, (4) one crosspoint per
# special row between start and end, and (5) crosspoint scores equal to the
# Stage-1 special rows (H, or F for a gap).

NEGI = -(1 << 40)


def _segment_score(a, b, ma, mi, go, ge, t_s, t_e):
    """Best global score of a[0:] x b[0:] as a segment between two crosspoints:
    t_s = 2 -> must start by continuing a vertical gap (G_ext per row, no
    opening); t_e = 2 -> must end with a vertical gap into the end cell."""
    gf = go + ge
    m, n = len(a), len(b)
    H = [[NEGI] * (n + 1) for _ in range(m + 1)]
    E = [[NEGI] * (n + 1) for _ in range(m + 1)]
    F = [[NEGI] * (n + 1) for _ in range(m + 1)]
    if t_s == 0:
        H[0][0] = 0
        for j in range(1, n + 1):
            H[0][j] = E[0][j] = -(go + j * ge)
        for i in range(1, m + 1):
            H[i][0] = F[i][0] = -(go + i * ge)
    else:  # continuing the vertical gap of the start crosspoint
        for i in range(1, m + 1):
            H[i][0] = F[i][0] = -i * ge
    for i in range(1, m + 1):
        for j in range(1, n + 1):
            E[i][j] = max(E[i][j - 1] - ge, H[i][j - 1] - gf)
            F[i][j] = max(F[i - 1][j] - ge, H[i - 1][j] - gf)
            p = ma if a[i - 1] == b[j - 1] else mi
            H[i][j] = max(E[i][j], F[i][j], H[i - 1][j - 1] + p)
    if t_e == 2:
        return F[m][n]
    return H[m][n]


def _check_stage2_list(A, B, sc, k):
    (best, ie, je), rows = oracle.stage1(A, B, *sc, k=k, keep_rows=True) if k > 0 else (oracle.stage1(A, B, *sc, k=0)[0], [])
    L = oracle.stage2(A, B, *sc, k, best, ie, je)
    assert L[-1] == (ie, je, best, 0)
    i1, j1, s1, t1 = L[0]
    assert (s1, t1) == (0, 0)
    # (3) the start point: the alignment from it to the end scores best
    assert oracle.global_score(A[i1:ie], B[j1:je], *sc) == best or best == 0
    # (4) one crosspoint per special row strictly between start and end
    if k > 0:
        want_rows = [r for r in range(k, ie, k) if r > i1]
        assert [c[0] for c in L[1:-1]] == want_rows
    # (5) scores are the special rows' H (type 0) or F (type 2)
    H = {r: h for r, h, f in rows}
    Fm = {r: f for r, h, f in rows}
    for (i, j, s, t) in L[1:-1]:
        if j == 0:
            assert (s, t) == (0, 0)
        else:
            assert s == (Fm[i][j - 1] if t == 2 else H[i][j - 1]), (i, j, s, t)
    # (2) partition additivity with the type-aware segment score
    for (cs, ce) in zip(L, L[1:]):
        seg = _segment_score(A[cs[0]:ce[0]], B[cs[1]:ce[1]], *sc, cs[3], ce[3])
        assert seg == ce[2] - cs[2], (cs, ce, seg)
    return L


def test_stage2_planted_gap_closed_forms():
    # X + TTTT + Y against X + Y: a 4-row vertical gap (a gap in S1) after
    # 20 matches.  Crossing row 20 + d (d = 1..3) inside the gap, the special
    # row's F is 20 - G_first - (d - 1) G_ext (Eq. 3); at row 24 the gap has
    # closed and the crosspoint is H-type with H = 20 - 3 - 4*2 = 9.
    X = "ACGTTGCAACGGTACCTGAT"
    Y = "GGCATTACGATCCAGTACGA"
    A, B = X + "TTTT" + Y, X + Y
    best = 40 - (3 + 4 * 2)
    assert oracle.stage1(A, B, *PAPER, k=0)[0] == (best, 44, 40)
    L = _check_stage2_list(A, B, PAPER, 22)
    assert L == [(0, 0, 0, 0), (22, 20, 20 - 5 - 2, 2), (44, 40, best, 0)]
    L1 = _check_stage2_list(A, B, PAPER, 1)
    assert L1[21:25] == [(21, 20, 15, 2), (22, 20, 13, 2), (23, 20, 11, 2), (24, 20, 9, 0)]
    assert all(c == (r, r, r, 0) for r, c in zip(range(21), L1[:21]))
    # no special row between start and end: the list is {start, end}
    assert _check_stage2_list(A, B, PAPER, 100) == [(0, 0, 0, 0), (44, 40, best, 0)]


@pytest.mark.parametrize("seed", range(6))
def test_stage2_properties_random(seed):
    rng = random.Random(seed)
    sc = [PAPER, (2, -1, 4, 1), (1, -1, 0, 2), (5, -4, 10, 1), (3, -2, 0, 1), (1, -3, 3, 2)][seed]
    A, B = synth.random_pair(300 + seed, 160 + 7 * seed, 150, plant_len=120, s=0.08, g=0.04, mu=3)
    A, B = A.tobytes().decode(), B.tobytes().decode()
    for k in (1, 3, 16, 40, 500):
        _check_stage2_list(A, B, sc, k)
    # an inserted/deleted block crossing several special rows
    base = _rand_seq(rng, 60)
    A2 = base[:30] + _rand_seq(rng, 9) + base[30:]
    _check_stage2_list(A2, base, sc, 4)
    _check_stage2_list(base, A2, sc, 4)


def test_stage2_zero_score_and_no_rows():
    assert oracle.stage2("AAAA", "CCCC", *PAPER, 2, 0, 0, 0) == [(0, 0, 0, 0)]
    (b, i, j), _ = oracle.stage1("ACGT", "ACGT", *PAPER, k=0)
    assert oracle.stage2("ACGT", "ACGT", *PAPER, 0, b, i, j) == [(0, 0, 0, 0), (4, 4, 4, 0)]
