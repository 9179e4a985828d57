#!/usr/bin/env python3
"""Time the full alignment (sw_align: Stages 1-5) against Stage 1 alone on a
workload: python tools/align_bench.py C2 [C1 C4 ...].  Prints the alignment
summary, wall times and the Stage 2-5 overhead."""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import synth  # noqa: E402
from paper_conf_ipps_sandesm11_b200 import Context  # noqa: E402

SC = (1, -3, 3, 2)
for wl in sys.argv[1:] or ["C2"]:
    cfg = synth.CONFIGS[wl]
    A, B = synth.make_pair(cfg)
    with Context(0) as ctx:
        ctx.align(A[:5000], B[:5000], *SC, k=64)  # warm-up
        t0 = time.perf_counter()
        r1, _ = ctx.align_stage1(A, B, *SC, k=cfg.k, sink=lambda *x: False)
        t1 = time.perf_counter()
        r = ctx.align(A, B, *SC, k=cfg.k)
        t2 = time.perf_counter()
        cells = len(A) * len(B)
        ngap = sum(g[2] for g in r["gap1"]) + sum(g[2] for g in r["gap2"])
        print(f"{wl}: score={r['score']} start={r['start']} end={r['end']} gap runs={len(r['gap1'])}+{len(r['gap2'])} "
              f"gap columns={ngap} partitions={r['partitions']} mm_levels={r['mm_levels']}")
        print(f"  sw_align_stage1 (rows to a Python sink) {1e3*(t1-t0):.1f} ms | sw_align {1e3*(t2-t1):.1f} ms: "
              + " ".join(f"{k} {v:.1f} ms" for k, v in r["ms"].items()), flush=True)
