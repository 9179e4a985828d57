#!/usr/bin/env python3
"""Debug: multi-device entries (virtual peers) in stripe and cyclic modes."""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("SWB_TIMEOUT_S", "5")
import numpy as np  # noqa: E402

import oracle  # noqa: E402
import synth  # noqa: E402
from paper_conf_ipps_sandesm11_b200 import Context  # noqa: E402

PAPER = (1, -3, 3, 2)
P = int(sys.argv[1]) if len(sys.argv) > 1 else 2
c = Context(devices=[0] * P)
A, B = synth.random_pair(8400, 9000, 40 * P + 1777, plant_len=1500, s=0.04, g=0.01)
want, orows = oracle.stage1(A.tobytes(), B.tobytes(), *PAPER, k=32)
for mode, variant, packed, grid in (("vstripes", 1, True, 0), ("mstr", 1, True, P), ("mstr", 1, True, 0), ("mstr", 1, False, 0),
                                    ("cyc", 1, True, 1), ("cyc-ring", 1, True, 1)):
    c.set_kernel(variant, packed)
    c.set_grid(grid)
    c.set_multi_gpu(mode.startswith("cyc"))
    c.set_row_budget(1 if mode == "cyc-ring" else 0)
    c.set_virtual_stripes(P if mode == "vstripes" else 1)
    t0 = time.time()
    try:
        got, rows = c.align_stage1(A, B, *PAPER, k=32, keep_rows=True)
        ok = got.astuple() == want and all(np.array_equal(h, oh) and np.array_equal(f, of)
                                           for (_, h, f), (_, oh, of) in zip(rows, orows))
        print(mode, variant, packed, grid, "ok" if ok else "MISMATCH", got.astuple(), want, c.stats(), f"{time.time()-t0:.2f}s", flush=True)
    except Exception as e:
        print(mode, variant, packed, grid, "ERROR", e, f"{time.time()-t0:.2f}s", flush=True)
c.set_virtual_stripes(1)
c.close()
