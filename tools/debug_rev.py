import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import oracle, synth
from paper_conf_ipps_sandesm11_b200 import Context
ctx = Context(0)
def s(x): return x.tobytes().decode() if isinstance(x, np.ndarray) else x
for seed in range(4):
    m, n = 300 + 411 * seed, 280 + 397 * seed
    A, B = synth.random_pair(100 + seed, m, n, plant_len=min(m, n) // 2, s=0.06, g=0.02)
    (sc, ie, je), _ = oracle.stage1(s(A), s(B), 1, -3, 3, 2)
    want = oracle.reverse_goal(s(A), ie, s(B), je, 1, -3, 3, 2, sc)
    for patch in (1, 0):
        ctx.set_patch(bool(patch))
        try:
            got = ctx.reverse_goal(A, ie, B, je, sc, 1, -3, 3, 2).astuple()
        except Exception as e:
            got = repr(e)
        print(seed, (m, n), "goal", sc, (ie, je), "patch", patch, "got", got, "want", want, ctx.stats()["alpha"], flush=True)
    ctx.set_patch(True)
