"""Compare the packed and int32 Stage-1 kernels cell by cell (k = 16 rows)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import synth
from paper_conf_ipps_sandesm11_b200 import Context

m, n = int(sys.argv[1]) if len(sys.argv) > 1 else 1100, int(sys.argv[2]) if len(sys.argv) > 2 else 300
A, B = synth.random_pair(1016, m, n, plant_len=min(m, n) // 2, s=0.08)
os.environ["SWB_PACKED"] = "0"; c32 = Context(0)
os.environ["SWB_PACKED"] = "1"; c16 = Context(0)
r32, rows32 = c32.align_stage1(A, B, 1, -3, 3, 2, k=16, keep_rows=True)
r16, rows16 = c16.align_stage1(A, B, 1, -3, 3, 2, k=16, keep_rows=True)
print("best int32", r32, "packed", r16, c16.stats()["alpha"])
for (r, h, f), (_, h2, f2) in zip(rows32, rows16):
    dh = np.flatnonzero(h != h2); df = np.flatnonzero(f != f2)
    if len(dh) or len(df):
        j = min(list(dh[:1]) + list(df[:1]))
        print("first diff row", r, "col", j + 1, "H", h[j:j+6], h2[j:j+6], "F", f[j:j+6], f2[j:j+6], "ndiff", len(dh), len(df))
        break
else:
    print("all special rows equal")
