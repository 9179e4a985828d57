"""oracle -- TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously-correct CPU implementation of CUDAlign 2.0 Stage 1
(Sandes & de Melo, IPDPS 2011; ``/root/reference/PAPER.md`` = ``P:<line>``):
Smith-Waterman with Gotoh affine gaps (Eq. 1-3), best score and its
end cell, special rows of H and F, and the anchored
global reverse pass used to find the start cell.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import this package.  It shares no code with
the CUDA path (``paper_conf_ipps_sandesm11_b200``) and imports nothing from
it; the only module both sides use is ``synth`` (seeded inputs, none of the
method's arithmetic).

Functions (all scores in the API convention: ``match``/``mismatch`` are added,
``gap_open``/``gap_ext`` are non-negative penalties that are subtracted,
G_first = gap_open + gap_ext, reading S2 in DESIGN.md):

- ``stage1(A, B, ma, mi, go, ge, k=0)`` -> ``(score, i, j), rows``
- ``full_matrix(A, B, ...)`` -> ``H, E, F`` (numpy int64, (m+1) x (n+1))
- ``band(A, B, ..., r0, r1, Htop, Ftop)`` -> ``Hbot, Fbot, (score, i, j)``
- ``global_score(A, B, ...)`` -> NW/Gotoh global score
- ``reverse_goal(A, i_end, B, j_end, ..., goal)`` -> ``(goal, i_s, j_s)`` or None
- ``flush_rows(m, n, alphaT, sra_bytes)`` -> special-row spacing
- ``stage2(A, B, ..., k, best, i_end, j_end)`` -> crosspoint list L_2
- ``align_partition(A, B, ..., Cs, Ce)`` -> (score, moves) of one partition
- ``align(A, B, ..., k)`` -> the full optimal local alignment (Stages 1, 2, then
  one partition at a time) with its GAP_1 / GAP_2 lists

Parity pins live in ``tests/test_oracle_pins.py``; every function above is
pinned (none is "parity unpinned").
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "sw_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

NEG = -(1 << 40)  # the oracle's "minus infinity" (sw_oracle.c)


class _Res(ctypes.Structure):
    _fields_ = [("score", ctypes.c_int64), ("i", ctypes.c_int64), ("j", ctypes.c_int64)]


_SINK = ctypes.CFUNCTYPE(
    ctypes.c_int,
    ctypes.c_void_p,
    ctypes.c_int64,
    ctypes.POINTER(ctypes.c_int64),
    ctypes.POINTER(ctypes.c_int64),
    ctypes.c_int64,
)


def build(force: bool = False) -> str:
    """Compile sw_oracle.c with gcc (plain -O2, no vectorisation pragmas)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is None:
            lib = ctypes.CDLL(build())
            i64, cp, vp = ctypes.c_int64, ctypes.c_char_p, ctypes.c_void_p
            p64 = ctypes.POINTER(ctypes.c_int64)
            lib.or_stage1.argtypes = [cp, i64, cp, i64, i64, i64, i64, i64, i64, _SINK, vp, ctypes.POINTER(_Res)]
            lib.or_full_matrix.argtypes = [cp, i64, cp, i64, i64, i64, i64, i64, p64, p64, p64]
            lib.or_band.argtypes = [cp, i64, cp, i64, i64, i64, i64, i64, i64, i64, p64, p64, p64, p64, ctypes.POINTER(_Res)]
            lib.or_global.argtypes = [cp, i64, cp, i64, i64, i64, i64, i64]
            lib.or_global.restype = i64
            lib.or_reverse_goal.argtypes = [cp, i64, cp, i64, i64, i64, i64, i64, i64, ctypes.POINTER(_Res)]
            lib.or_stage2.argtypes = [cp, i64, cp, i64, i64, i64, i64, i64, i64, i64, i64, i64, p64, i64]
            lib.or_stage2.restype = i64
            lib.or_align_partition.argtypes = [cp, cp, i64, i64, i64, i64, i64, i64, i64, i64, i64, i64,
                                               ctypes.c_char_p, i64, p64]
            lib.or_align_partition.restype = i64
            lib.or_flush_rows.argtypes = [i64, i64, i64, i64]
            lib.or_flush_rows.restype = i64
            _lib = lib
    return _lib


def _b(s) -> bytes:
    if isinstance(s, np.ndarray):
        return s.tobytes()
    if isinstance(s, str):
        return s.encode("ascii")
    return bytes(s)


def _p64(a: np.ndarray):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_int64))


def stage1(A, B, ma, mi, go, ge, k=0, sink=None, keep_rows=True):
    """Stage 1.  Returns ((score, i, j), rows) where rows is a list
    of (i, H[1..n], F[1..n]) for every special row (if keep_rows), and calls
    ``sink(i, H, F)`` (numpy int64 copies) for each if given."""
    lib = _load()
    a, b = _b(A), _b(B)
    rows = []

    def _cb(_user, row, H, F, n):
        h = np.ctypeslib.as_array(H, shape=(n,)).copy()
        f = np.ctypeslib.as_array(F, shape=(n,)).copy()
        if keep_rows:
            rows.append((int(row), h, f))
        if sink is not None:
            return int(bool(sink(int(row), h, f)))
        return 0

    cb = _SINK(_cb)
    res = _Res()
    rc = lib.or_stage1(a, len(a), b, len(b), ma, mi, go, ge, k, cb, None, ctypes.byref(res))
    if rc != 0:
        raise RuntimeError(f"or_stage1 failed rc={rc}")
    return (res.score, res.i, res.j), rows


def full_matrix(A, B, ma, mi, go, ge):
    lib = _load()
    a, b = _b(A), _b(B)
    m, n = len(a), len(b)
    H = np.zeros((m + 1, n + 1), np.int64)
    E = np.zeros_like(H)
    F = np.zeros_like(H)
    lib.or_full_matrix(a, m, b, n, ma, mi, go, ge, _p64(H), _p64(E), _p64(F))
    return H, E, F


def band(A, B, ma, mi, go, ge, r0, r1, Htop, Ftop):
    """Rows r0+1..r1 from row r0 (each length n+1, column 0 included)."""
    lib = _load()
    a, b = _b(A), _b(B)
    n = len(b)
    Ht = np.ascontiguousarray(Htop, dtype=np.int64)
    Ft = np.ascontiguousarray(Ftop, dtype=np.int64)
    assert Ht.shape == (n + 1,) and Ft.shape == (n + 1,)
    Hb = np.zeros(n + 1, np.int64)
    Fb = np.zeros(n + 1, np.int64)
    res = _Res()
    rc = lib.or_band(a, len(a), b, n, ma, mi, go, ge, r0, r1, _p64(Ht), _p64(Ft), _p64(Hb), _p64(Fb), ctypes.byref(res))
    if rc != 0:
        raise RuntimeError(f"or_band failed rc={rc}")
    return Hb, Fb, (res.score, res.i, res.j)


def global_score(A, B, ma, mi, go, ge) -> int:
    lib = _load()
    a, b = _b(A), _b(B)
    return int(lib.or_global(a, len(a), b, len(b), ma, mi, go, ge))


def reverse_goal(A, i_end, B, j_end, ma, mi, go, ge, goal):
    lib = _load()
    a, b = _b(A), _b(B)
    res = _Res()
    found = lib.or_reverse_goal(a, i_end, b, j_end, ma, mi, go, ge, goal, ctypes.byref(res))
    return (res.score, res.i, res.j) if found else None


def stage2(A, B, ma, mi, go, ge, k, best, i_end, j_end):
    """Stage 2 crosspoint list L_2, ascending: [(i, j, score, type), ...]
    from the start point to the end point (i_end, j_end, best, 0); type 2 = vertical gap."""
    lib = _load()
    a, b = _b(A), _b(B)
    cap = 64
    while True:
        buf = (ctypes.c_int64 * (4 * cap))()
        cnt = lib.or_stage2(a, len(a), b, len(b), ma, mi, go, ge, k, best, i_end, j_end,
                            ctypes.cast(buf, ctypes.POINTER(ctypes.c_int64)), cap)
        if cnt < 0:
            raise RuntimeError(f"or_stage2 failed rc={cnt}")
        if cnt <= cap:
            return [tuple(int(buf[4 * q + x]) for x in range(4)) for q in range(cnt)]
        cap = cnt


def flush_rows(m, n, alphaT, sra_bytes) -> int:
    return int(_load().or_flush_rows(m, n, alphaT, sra_bytes))


def align_partition(A, B, ma, mi, go, ge, Cs, Ce):
    """Optimal alignment of partition (Cs, Ce), Cs = (i_s, j_s, type_s),
    Ce = (i_e, j_e, type_e); types 0 any / 1 horizontal gap (E) / 2 vertical gap (F).
    Returns (score, moves) with moves a str over 'M' (pair), 'I' (gap in S0),
    'D' (gap in S1), or (None, None) if no alignment has these end states."""
    lib = _load()
    a, b = _b(A), _b(B)
    (i_s, j_s, t_s), (i_e, j_e, t_e) = Cs, Ce
    cap = max(0, (i_e - i_s) + (j_e - j_s))
    buf = ctypes.create_string_buffer(cap + 1)
    nops = ctypes.c_int64(0)
    sc = lib.or_align_partition(a, b, i_s, j_s, i_e, j_e, ma, mi, go, ge, t_s, t_e, buf, cap, ctypes.byref(nops))
    if sc <= NEG // 2:
        return None, None
    if nops.value < 0:
        raise RuntimeError("or_align_partition failed")
    return int(sc), buf.raw[: nops.value].decode()


def gap_lists(moves, i0, j0):
    """GAP_1 / GAP_2 of P:281 from a move string starting at DP cell (i0, j0):
    (i, j, length) per maximal gap run, (i, j) the cell the run leaves from
    (reading S24).  GAP_1 = gaps in S0 (horizontal, 'I'), GAP_2 = gaps in S1
    (vertical, 'D')."""
    g1, g2 = [], []
    i, j, q = i0, j0, 0
    while q < len(moves):
        c = moves[q]
        r = q
        while r < len(moves) and moves[r] == c:
            r += 1
        L = r - q
        if c == "M":
            i += L
            j += L
        elif c == "I":
            g1.append((i, j, L))
            j += L
        else:
            g2.append((i, j, L))
            i += L
        q = r
    return g1, g2


def align(A, B, ma, mi, go, ge, k):
    """The full optimal local alignment: Stage 1 (best, end point, special rows
    every k rows), Stage 2 (crosspoints L_2), then every partition between
    consecutive crosspoints aligned on its own (Stages 3-5 reach the same
    partition alignments in linear space).  Returns a dict with
    score, start (i0, j0), end (i1, j1), moves, gap1, gap2, crosspoints."""
    (best, ie, je), _ = stage1(A, B, ma, mi, go, ge, k=0, keep_rows=False)
    if best == 0:
        return {"score": 0, "start": (0, 0), "end": (0, 0), "moves": "", "gap1": [], "gap2": [], "crosspoints": []}
    L = stage2(A, B, ma, mi, go, ge, k, best, ie, je)
    moves = []
    for (i_s, j_s, sc_s, t_s), (i_e, j_e, sc_e, t_e) in zip(L, L[1:]):
        sc, mv = align_partition(A, B, ma, mi, go, ge, (i_s, j_s, t_s), (i_e, j_e, t_e))
        if sc != sc_e - sc_s:
            raise RuntimeError(f"partition {(i_s, j_s, t_s)} -> {(i_e, j_e, t_e)}: {sc} != {sc_e - sc_s}")
        moves.append(mv)
    mv = "".join(moves)
    g1, g2 = gap_lists(mv, L[0][0], L[0][1])
    return {"score": best, "start": (L[0][0], L[0][1]), "end": (ie, je), "moves": mv, "gap1": g1, "gap2": g2,
            "crosspoints": L}
