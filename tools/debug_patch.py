import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth
from paper_conf_ipps_sandesm11_b200 import Context
ctx = Context(0)
for v, (m, n) in [(0, (1, 1)), (0, (1, 1)), (0, (100, 100)), (-1, (100, 100)), (8, (300, 300)), (0, (17, 1))]:
    ctx.set_kernel(v, True)
    A, B = synth.random_pair(1, m, n, plant_len=min(m, n) // 2)
    r, _ = ctx.align_stage1(A, B, 1, -3, 3, 2, k=32, keep_rows=True)
    st = ctx.stats()
    print(v, m, n, r.astuple(), "alpha", st["alpha"], "patched", st["patched"], "err", ctx._lib.sw_last_error(ctx._h), flush=True)
