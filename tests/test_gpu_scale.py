"""Parity at BASELINE.json sizes, in the launch configuration bench.py times.

The oracle cannot redo 1e11-1e13 cells in one thread inside a test, so the
GPU's output is checked by band induction:
row 0 is trivially correct; for every band [r, r + k) the oracle recomputes
rows r+1..r+k from the GPU's special row r and must reproduce the GPU's
special row r + k bit for bit, and the band maxima (oracle-computed) combine
under (max, min i, min j) into the GPU's best cell.  Bands run in parallel on
the host cores.  C2 is checked completely (every row, the global best); C3 is
checked on a seeded sample of bands plus the band that holds the end cell.
"""
import os
from multiprocessing.pool import ThreadPool

import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu
PAPER = (1, -3, 3, 2)

_G = {}


def _band_job(args):
    q, r0, r1 = args
    A, B, rows = _G["A"], _G["B"], _G["rows"]
    n = len(B)
    if r0 == 0:
        Ht = np.zeros(n + 1, np.int64)
        Ft = np.full(n + 1, oracle.NEG, np.int64)
    else:
        h, f = rows[r0]
        Ht = np.concatenate([[0], h.astype(np.int64)])
        Ft = np.concatenate([[oracle.NEG], f.astype(np.int64)])
    Hb, Fb, best = oracle.band(A, B, *PAPER, r0, r1, Ht, Ft)
    ok = True
    if r1 in rows:
        h, f = rows[r1]
        ok = bool(np.array_equal(Hb[1:], h) and np.array_equal(Fb[1:], f))
    return q, ok, best


def _run_bands(A, B, rows, jobs):
    """Bands in parallel on the host cores: threads, since the oracle's C band
    loop runs inside a ctypes call that releases the GIL (no fork of this
    CUDA-initialised process)."""
    _G.update(A=A.tobytes(), B=B.tobytes(), rows=rows)
    oracle.build()
    with ThreadPool(min(len(jobs), os.cpu_count() or 4)) as pool:
        return pool.map(_band_job, jobs, chunksize=1)


@pytest.fixture(scope="module")
def ctx():
    from paper_conf_ipps_sandesm11_b200 import Context, build

    build.build()
    c = Context(0)
    yield c
    c.close()


def test_c2_full_band_induction(ctx):
    """BASELINE configs[1] (543K x 536K, k = 3840): every special row and the
    best cell, bit-exact, plus the reverse-pass start cell."""
    cfg = synth.CONFIGS["C2"]
    A, B = synth.make_pair(cfg)
    rows = {}

    def sink(row, H, F):
        rows[row] = (H.copy(), F.copy())

    got, _ = ctx.align_stage1(A, B, *PAPER, k=cfg.k, sink=sink)
    # the kernel bench.py times: the alpha-30 packed geometry (142 bands of 3840 rows)
    s1 = ctx.stats()
    assert (s1["alpha"], s1["warps"], s1["grid"], s1["patched"]) == (-30, 4, 142, 1), s1
    assert sorted(rows) == list(range(cfg.k, cfg.m + 1, cfg.k))
    bounds = list(range(0, cfg.m, cfg.k)) + [cfg.m]
    jobs = [(q, bounds[q], bounds[q + 1]) for q in range(len(bounds) - 1)]
    res = _run_bands(A, B, rows, jobs)
    assert all(ok for _, ok, _ in res), [q for q, ok, _ in res if not ok]
    bests = [b for _, _, b in res if b[0] > 0]
    want = max(bests, key=lambda x: (x[0], -x[1], -x[2]))
    assert got.astuple() == want
    # the reverse pass from the end cell, against the oracle
    st = ctx.reverse_goal(A, got.i, B, got.j, got.score, *PAPER)
    assert st.astuple() == oracle.reverse_goal(A.tobytes(), got.i, B.tobytes(), got.j, *PAPER, got.score)
    assert (st.i, st.j) == (cfg.params["a0"], cfg.params["b0"])  # the planted segment's start (Table III shape)


def _sampled_induction(ctx, cfg, k, sample, expect_kernel):
    """Stage 1 of `cfg` at special-row spacing k; the oracle recomputes the
    sampled bands [q k, (q + 1) k) from the GPU's row q k and must reproduce row
    (q + 1) k bit for bit; the band holding the end cell must hold the best."""
    A, B = synth.make_pair(cfg)
    keep = set()
    for q in sample:
        keep.update({q * k, (q + 1) * k})
    rows = {}

    def sink(row, H, F):
        if row in keep:
            rows[row] = (H.copy(), F.copy())

    got, _ = ctx.align_stage1(A, B, *PAPER, k=k, sink=sink)
    s1 = ctx.stats()
    if expect_kernel is not None:
        assert (s1["alpha"], s1["warps"], s1["patched"]) == expect_kernel, s1
    else:  # the automatic choice (the one bench.py runs): a patched packed geometry, maybe with a tail segment
        assert s1["alpha"] < 0 and s1["patched"] == 1, s1
    assert s1["special_rows"] == cfg.m // k
    jobs = [(q, q * k, min((q + 1) * k, cfg.m)) for q in sorted(sample) if q * k < cfg.m]
    res = _run_bands(A, B, rows, jobs)
    assert all(ok for _, ok, _ in res), [q for q, ok, _ in res if not ok]
    qe = (got.i - 1) // k
    assert qe in sample, (qe, sorted(sample))
    band_best = {q: b for q, _, b in res}[qe]
    assert band_best == got.astuple()
    # no sampled band may hold a better cell than the reported best (the total order)
    for q, _, b in res:
        assert b[0] < got.score or (b[0] == got.score and (b[1], b[2]) >= (got.i, got.j)), (q, b, got)
    return got


def test_c3_sampled_band_induction(ctx):
    """C3 (5M x 5M, whole-length homology) in the geometry its bench line runs
    (alpha 16 x 8 warps, 1221 bands of 4096 rows on 148 CTAs: 8+ waves):
    special rows every 4096 rows (one per band, drained by the I/O warp); a
    seeded sample of bands plus the last full band and the ragged tail, where
    the end cell lies."""
    cfg = synth.CONFIGS["C3"]
    k = 4096
    rng = np.random.default_rng(3)
    nbands = cfg.m // k
    sample = set(int(x) for x in rng.choice(nbands, size=10, replace=False))
    sample.update({nbands - 1, nbands})
    got = _sampled_induction(ctx, cfg, k, sample, (-16, 8, 1))
    assert got.i > cfg.m - 2 * k  # whole-length alignment ends near the corner


def test_c4_sampled_band_induction(ctx):
    """C4 (10M x 10M, the scaling config) in the geometry bench.py times (the
    automatic choice: several waves of tall bands, plus a tail segment when the
    last wave is partial): special rows every 8192 rows; a
    seeded sample of bands from every wave, the bands around the planted
    homology (the end cell) and the ragged last band."""
    cfg = synth.CONFIGS["C4"]
    k = 8192
    rng = np.random.default_rng(4)
    nbands = cfg.m // k
    sample = set(int(x) for x in rng.choice(nbands, size=4, replace=False))
    a0, L = cfg.params["a0"], cfg.params["L"]
    sample.update(range(a0 // k, (a0 + 2 * L) // k + 1))
    sample.add(nbands)  # the ragged last band
    got = _sampled_induction(ctx, cfg, k, sample, None)
    assert a0 < got.i <= a0 + 2 * L
