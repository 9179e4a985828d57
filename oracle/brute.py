"""oracle.brute -- TEST INFRASTRUCTURE ONLY.

Dynamic-programming-free definitions for tiny inputs (m, n <= ~6), used to
pin the C oracle.  Every alignment path is enumerated explicitly and scored
column by column with the affine gap model of P:50: a maximal run of L gap
columns of the same kind costs G_first + (L-1) G_ext, G_first = G_open + G_ext
(reading S2), a pair column scores ma / mi (reading S1).

A path starts at a DP cell (s, t) with value 0 (the local alignment's
"start", reading S8: the cell before the first aligned pair) and moves with
three ops:
  'D' diagonal: aligns S0[i+1] with S1[j+1]
  'H' horizontal: S1[j+1] against a gap (the E matrix, Eq. 2)
  'V' vertical:   S0[i+1] against a gap (the F matrix, Eq. 3)

From these paths, for every cell (i, j):
  E(i,j) = max score of a path ending at (i,j) whose last op is 'H'
  F(i,j) = max score of a path ending at (i,j) whose last op is 'V'
  H(i,j) = max(0, every path ending at (i,j))
which is what Eq. 1-3 compute (Gotoh) -- but here as a maximum
over explicitly listed alignments, not a recurrence.
"""
from __future__ import annotations

NEG = None  # "no path"


def _mx(a, b):
    if a is None:
        return b
    if b is None:
        return a
    return a if a >= b else b


def local_matrices(S0: str, S1: str, ma: int, mi: int, G_open: int, G_ext: int):
    """Return H, E, F as lists of lists (None = -infinity) for local mode."""
    m, n = len(S0), len(S1)
    G_first = G_open + G_ext
    H = [[0] * (n + 1) for _ in range(m + 1)]
    E = [[None] * (n + 1) for _ in range(m + 1)]
    F = [[None] * (n + 1) for _ in range(m + 1)]

    def walk(i, j, score, last):
        # record the path that ends here (non-empty paths only)
        if last == "D":
            H[i][j] = max(H[i][j], score)
        elif last == "H":
            E[i][j] = _mx(E[i][j], score)
            H[i][j] = max(H[i][j], score)
        elif last == "V":
            F[i][j] = _mx(F[i][j], score)
            H[i][j] = max(H[i][j], score)
        if i < m and j < n:
            p = ma if S0[i].upper() == S1[j].upper() else mi
            walk(i + 1, j + 1, score + p, "D")
        if j < n:
            walk(i, j + 1, score - (G_ext if last == "H" else G_first), "H")
        if i < m:
            walk(i + 1, j, score - (G_ext if last == "V" else G_first), "V")

    for s in range(m + 1):
        for t in range(n + 1):
            walk(s, t, 0, None)
    return H, E, F


def local_best(S0: str, S1: str, ma: int, mi: int, G_open: int, G_ext: int):
    """(score, i, j): the highest H, then smallest i, then smallest j (reading S4);
    (0, 0, 0) when no alignment scores above 0."""
    H, _, _ = local_matrices(S0, S1, ma, mi, G_open, G_ext)
    best = (0, 0, 0)
    for i in range(1, len(S0) + 1):
        for j in range(1, len(S1) + 1):
            if H[i][j] > best[0]:
                best = (H[i][j], i, j)
    return best


def score_alignment(top: str, bottom: str, ma: int, mi: int, G_open: int, G_ext: int) -> int:
    """Score a printed alignment column by column (Figure 1).
    '-' marks a gap; a maximal run of L gap columns in the same row costs
    G_first + (L-1) G_ext."""
    assert len(top) == len(bottom)
    G_first = G_open + G_ext
    s = 0
    prev = None
    for a, b in zip(top, bottom):
        if a == "-" and b == "-":
            raise ValueError("column with two gaps")
        if a == "-":
            s -= G_ext if prev == "top" else G_first
            prev = "top"
        elif b == "-":
            s -= G_ext if prev == "bottom" else G_first
            prev = "bottom"
        else:
            s += ma if a.upper() == b.upper() else mi
            prev = None
    return s


def global_best(S0: str, S1: str, ma: int, mi: int, G_open: int, G_ext: int) -> int:
    """Max score over all global alignments of S0 and S1 (NW), each
    listed explicitly (tiny inputs only)."""
    m, n = len(S0), len(S1)
    G_first = G_open + G_ext
    best = [None]

    def walk(i, j, score, last):
        if i == m and j == n:
            best[0] = _mx(best[0], score)
            return
        # Branch and bound (prunes, never changes the maximum): the rest of
        # any alignment scores at most min(ri, rj)*max(ma, 0) - |ri - rj|*G_ext,
        # since every gap column costs at least G_ext.
        ri, rj = m - i, n - j
        if best[0] is not None and score + min(ri, rj) * max(ma, 0) - abs(ri - rj) * G_ext <= best[0]:
            return
        if i < m and j < n:
            p = ma if S0[i].upper() == S1[j].upper() else mi
            walk(i + 1, j + 1, score + p, "D")
        if j < n:
            walk(i, j + 1, score - (G_ext if last == "H" else G_first), "H")
        if i < m:
            walk(i + 1, j, score - (G_ext if last == "V" else G_first), "V")

    walk(0, 0, 0, None)
    return best[0]


def all_local_starts(S0: str, S1: str, ma: int, mi: int, G_open: int, G_ext: int, i_end: int, j_end: int, goal: int):
    """Every start cell (s, t) from which some alignment path ending with a
    pair at (i_end, j_end) scores exactly `goal` (tiny inputs)."""
    G_first = G_open + G_ext
    starts = set()
    for s in range(i_end):
        for t in range(j_end):
            found = [False]

            def walk(i, j, score, last):
                if found[0] or i > i_end or j > j_end:
                    return
                if i == i_end and j == j_end and last == "D" and score == goal:
                    found[0] = True
                    return
                if i < i_end and j < j_end:
                    p = ma if S0[i].upper() == S1[j].upper() else mi
                    walk(i + 1, j + 1, score + p, "D")
                if j < j_end:
                    walk(i, j + 1, score - (G_ext if last == "H" else G_first), "H")
                if i < i_end:
                    walk(i + 1, j, score - (G_ext if last == "V" else G_first), "V")

            walk(s, t, 0, None)
            if found[0]:
                starts.add((s, t))
    return starts


def partition_best(S0: str, S1: str, ma: int, mi: int, G_open: int, G_ext: int, type_s: int, type_e: int):
    """Max score over all alignments of the whole of S0 with the whole of S1
    that start in crosspoint state type_s and end in state type_e:
    type 1 = the path is inside a horizontal gap (a gap in S0), type 2 = inside
    a vertical gap (a gap in S1), 0 = no constraint.  A gap run that continues
    the start state costs G_ext per column (its opening was charged before the
    partition); every other maximal run costs G_first + (L-1) G_ext.
    Each alignment is listed explicitly (tiny inputs only).  None if no
    alignment has the required end state."""
    m, n = len(S0), len(S1)
    G_first = G_open + G_ext
    best = [None]
    start_last = {0: None, 1: "H", 2: "V"}[type_s]
    want_last = {0: None, 1: "H", 2: "V"}[type_e]

    def walk(i, j, score, last):
        if i == m and j == n and (want_last is None or last == want_last):
            best[0] = _mx(best[0], score)
        if i < m and j < n:
            p = ma if S0[i].upper() == S1[j].upper() else mi
            walk(i + 1, j + 1, score + p, "D")
        if j < n:
            walk(i, j + 1, score - (G_ext if last == "H" else G_first), "H")
        if i < m:
            walk(i + 1, j, score - (G_ext if last == "V" else G_first), "V")

    walk(0, 0, 0, start_last)
    return best[0]
