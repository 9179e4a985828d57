"""Multi-device contexts through the C ABI (sw_init with n_devices > 1;
VERDICT r01 item 4), bit-exact against the oracle.

The round's GPU box has one B200, so the entries are "virtual peers": the
same device id repeated, each entry with its own streams, buffers and launch,
sharing the GPU's SMs.  The protocol is the one real peers run over NVLink:
band-cyclic Stage 1 (entry d takes bands d, d + P, ...; each band's bottom row
and progress go to the next entry's memory) or one column stripe per entry
(the (t, E) border column goes to the next entry's receive area), and the
library combines the entries' best cells (reading S4) and hands the sink whole
special rows.
"""
import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu
PAPER = (1, -3, 3, 2)


def _s(x):
    return x.tobytes().decode() if isinstance(x, np.ndarray) else x


@pytest.fixture(scope="module", params=[2, 4, 8])
def mctx(request):
    from paper_conf_ipps_sandesm11_b200 import Context, build

    build.build()
    c = Context(devices=[0] * request.param)
    yield c
    c.close()


def compare(got, rows, A, B, scoring, k):
    want, orows = oracle.stage1(_s(A), _s(B), *scoring, k=k)
    assert got.astuple() == want
    assert [r for r, _, _ in rows] == [r for r, _, _ in orows]
    for (r, h, f), (_, oh, of) in zip(rows, orows):
        assert np.array_equal(h, oh), f"H row {r}"
        assert np.array_equal(f, of), f"F row {r}"


def run(c, A, B, scoring, k, variant=-1, packed=True, cyclic=True, grid=0, budget=0):
    c.set_kernel(variant, packed)
    c.set_multi_gpu(cyclic)
    c.set_grid(grid)
    c.set_row_budget(budget)
    try:
        got, rows = c.align_stage1(A, B, *scoring, k=k, keep_rows=True)
        st = c.stats()
    finally:
        c.set_kernel(-1, True)
        c.set_multi_gpu(True)
        c.set_grid(0)
        c.set_row_budget(0)
    return got, rows, st


def test_device_count(mctx):
    assert mctx.device_count() == len(mctx.devices)


@pytest.mark.parametrize("variant,packed,alpha,nw", [(1, True, 16, 8), (10, True, 32, 8), (13, True, 30, 4),
                                                     (14, True, 34, 8), (1, False, 16, 8), (0, False, 16, 4)])
def test_cyclic_bands(mctx, variant, packed, alpha, nw):
    """Band-cyclic Stage 1: every entry runs bands, several per CTA at a small
    grid; special rows at strip bottoms (packed) or every row (int32)."""
    P = mctx.device_count()
    bh = alpha * 32 * nw
    m, n = 3 * P * bh // 2 + 333, (1200 if packed else 300)
    A, B = synth.random_pair(8000 + 10 * variant + P, m, n, plant_len=1000, s=0.04, g=0.01)
    k = alpha if packed else 1
    got, rows, st = run(mctx, A, B, PAPER, k, variant, packed, grid=1)
    assert st["devices"] == P and st["alpha"] == (-alpha if packed else alpha), st
    compare(got, rows, A, B, PAPER, k)


def test_cyclic_alpha34_staged_rows(mctx):
    """The geometry band-cyclic C4 runs on several GPUs (alpha 34 x 8 warps)
    with special rows that are neither strip nor band bottoms (k = band height
    + 5: the band-uniform staged tiles of the GEN kernel), bands of every entry."""
    P = mctx.device_count()
    k = 8704 + 5
    A, B = synth.random_pair(8200 + P, 3 * k + 111, 700, plant_len=1500, s=0.04, g=0.01)
    got, rows, st = run(mctx, A, B, PAPER, k, 14, True, grid=1)
    assert st["devices"] == P and st["alpha"] == -34, st
    compare(got, rows, A, B, PAPER, k)


def test_cyclic_auto_and_scorings(mctx):
    A, B = synth.random_pair(8100, 40000, 3000, plant_len=2500, s=0.03, g=0.01)
    for scoring in (PAPER, (2, -1, 4, 1), (5, -4, 10, 1), (100, -20, 20, 5)):
        got, rows, st = run(mctx, A, B, scoring, 960)
        assert st["devices"] == mctx.device_count(), st
        compare(got, rows, A, B, scoring, 960)


def test_cyclic_ties_across_entries(mctx):
    """Equal maxima in bands of different entries: the smallest row wins."""
    X = synth.random_pair(8200, 300, 1)[0]
    fill = synth.random_pair(8201, 9000, 1)[0]
    A = np.concatenate([fill[:4000], X, fill, X, fill[:100], X])
    got, rows, st = run(mctx, A, X, PAPER, 16, 1, True, grid=1)
    compare(got, rows, A, X, PAPER, 16)
    assert got.i == 4300


def test_cyclic_with_ring(mctx):
    """Band-cyclic with a minimal special-row ring per entry (back-pressure
    across entries)."""
    A, B = synth.random_pair(8300, 30000, 1500, plant_len=1200, s=0.04, g=0.01)
    got, rows, st = run(mctx, A, B, PAPER, 32, 1, True, grid=1, budget=1)
    assert st["sp_slots"] < 30000 // 32, st
    compare(got, rows, A, B, PAPER, 32)


@pytest.mark.parametrize("variant,packed", [(1, True), (1, False), (10, True)])
def test_entry_column_stripes(mctx, variant, packed):
    """One column stripe per entry: the (t, E) border column of every band goes
    to the next entry's receive area."""
    P = mctx.device_count()
    A, B = synth.random_pair(8400 + variant, 9000, 40 * P + 1777, plant_len=1500, s=0.04, g=0.01)
    k = 32 if packed else 7
    got, rows, st = run(mctx, A, B, PAPER, k, variant, packed, cyclic=False, grid=P)
    assert st["devices"] == P, st
    compare(got, rows, A, B, PAPER, k)


def test_other_stages_on_primary(mctx):
    """The reverse pass, Stage 2 and the full alignment run on entry 0; Stage 2
    reads the special rows of a band-cyclic Stage 1 from the host store."""
    A, B = synth.random_pair(8500, 7000, 6500, plant_len=6000, s=0.03, g=0.01)
    k = 256
    best, _ = mctx.align_stage1(A, B, *PAPER, k=k)
    want = oracle.stage1(_s(A), _s(B), *PAPER, k=0)[0]
    assert best.astuple() == want
    L2 = mctx.stage2(A, B, *PAPER, k=k, end=best)
    assert L2 == oracle.stage2(_s(A), _s(B), *PAPER, k, *want)
    st = mctx.reverse_goal(A, best.i, B, best.j, best.score, *PAPER)
    assert st.astuple() == oracle.reverse_goal(_s(A), best.i, _s(B), best.j, *PAPER, best.score)
    ra = mctx.align(A, B, *PAPER, k=k)
    wa = oracle.align(_s(A), _s(B), *PAPER, k)
    assert (ra["score"], ra["start"], ra["end"]) == (wa["score"], wa["start"], wa["end"])


def test_combine_best_in_library():
    from paper_conf_ipps_sandesm11_b200 import combine_best

    assert combine_best([(5, 9, 9), (5, 3, 7), (5, 3, 2), (4, 1, 1)]) == (5, 3, 2)
    assert combine_best([(0, 4, 4), (0, 0, 0)]) == (0, 0, 0)
    assert combine_best([]) == (0, 0, 0)
