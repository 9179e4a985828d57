#!/usr/bin/env python3
"""Debug: the special-row ring under a minimal budget (one case of tests/test_gpu_ring.py)."""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("SWB_TIMEOUT_S", "5")
os.environ.setdefault("SWB_DEBUG_HOST", "1")
import numpy as np  # noqa: E402

import oracle  # noqa: E402
import synth  # noqa: E402
from paper_conf_ipps_sandesm11_b200 import Context  # noqa: E402

PAPER = (1, -3, 3, 2)
c = Context(0)
variant, packed, grid, k = (int(x) for x in (sys.argv[1:] + ["1", "0", "1", "1"])[:4])
bh = 16 * 32 * 8
m, n = 3 * bh + 211, 777
A, B = synth.random_pair(6000 + variant + grid, m, n, plant_len=700, s=0.05, g=0.01)
c.set_kernel(variant, bool(packed))
c.set_grid(grid)
c.set_row_budget(1)
cnt = [0]


def sink(r, h, f):
    cnt[0] += 1


t0 = time.time()
try:
    got, rows = c.align_stage1(A, B, *PAPER, k=k, sink=sink)
    print("ok", got.astuple(), c.stats(), cnt[0], f"{time.time()-t0:.2f}s", flush=True)
except Exception as e:
    print("ERROR", e, cnt[0], f"{time.time()-t0:.2f}s", flush=True)
want, _ = oracle.stage1(A.tobytes(), B.tobytes(), *PAPER, k=0)
print("want", want)
