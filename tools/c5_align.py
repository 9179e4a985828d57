#!/usr/bin/env python3
"""The full alignment (sw_align: Stages 1-5) of a workload, once, with a
vectorised rescoring of the output alignment from its GAP_1/GAP_2 lists
(diagonal runs between gap runs): python tools/c5_align.py C5"""
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402
from paper_conf_ipps_sandesm11_b200 import Context  # noqa: E402

SC = (1, -3, 3, 2)
wl = sys.argv[1] if len(sys.argv) > 1 else "C5"
cfg = synth.CONFIGS[wl]
t0 = time.perf_counter()
A, B = synth.make_pair(cfg)
print(f"{wl}: {len(A)} x {len(B)} generated in {time.perf_counter() - t0:.1f} s", flush=True)
with Context(0) as ctx:
    ctx.align(A[:5000], B[:5000], *SC, k=64)  # warm-up
    t1 = time.perf_counter()
    r = ctx.align(A, B, *SC, k=cfg.k)
    t2 = time.perf_counter()
print(f"  score={r['score']} start={r['start']} end={r['end']} gap runs={len(r['gap1'])}+{len(r['gap2'])} "
      f"partitions={r['partitions']} mm_levels={r['mm_levels']}")
print(f"  sw_align {t2 - t1:.1f} s: " + " ".join(f"{k} {v / 1e3:.1f} s" for k, v in r["ms"].items()), flush=True)
# rescoring: events sorted by position; diagonal runs between them
ma, mi, go, ge = SC
ev = sorted([(gi, gj, L, 1) for gi, gj, L in r["gap1"]] + [(gi, gj, L, 2) for gi, gj, L in r["gap2"]])
i, j = r["start"]
score, gapcols, diag_i, diag_j, diag_len = 0, 0, [], [], []
for gi, gj, L, c in ev:
    d = gi - i
    assert d >= 0 and gj - j == d, (gi, gj, i, j)
    diag_i.append(i); diag_j.append(j); diag_len.append(d)
    score -= go + L * ge
    gapcols += L
    i, j = (gi, gj + L) if c == 1 else (gi + L, gj)
d = r["end"][0] - i
assert d >= 0 and r["end"][1] - j == d
diag_i.append(i); diag_j.append(j); diag_len.append(d)
matches = mism = 0
for a0, b0, L in zip(diag_i, diag_j, diag_len):
    if L:
        eq = int(np.count_nonzero(A[a0:a0 + L] == B[b0:b0 + L]))
        matches += eq; mism += L - eq
score += matches * ma + mism * mi
print(f"  rescored {score} ({'== score' if score == r['score'] else 'MISMATCH'}): {matches} matches, {mism} mismatches, "
      f"{len(ev)} gap runs, {gapcols} gap columns, length {matches + mism + gapcols}")
