"""Print where a fixed int32 variant's special rows differ from the oracle (debug aid)."""
import sys
import numpy as np
import oracle, synth
from paper_conf_ipps_sandesm11_b200 import Context

v = int(sys.argv[1])
ctx = Context(0)
A, B = synth.random_pair(50 + v, 2600, 1900, plant_len=1500, s=0.06, g=0.01)
S = lambda x: x.tobytes().decode()
for scoring, k in (((1, -3, 3, 2), 7), ((2, -1, 4, 1), 32), ((1, -1, 0, 2), 0), ((100, -20, 20, 5), 100)):
    ctx.set_kernel(v, False)
    got, rows = ctx.align_stage1(A, B, *scoring, k=k, keep_rows=True)
    want, orows = oracle.stage1(S(A), S(B), *scoring, k=k)
    print(scoring, k, got.astuple(), want, len(rows), len(orows))
    nbad = 0
    for (r, h, f), (_, oh, of) in zip(rows, orows):
        bh = np.nonzero(h != oh)[0]
        bf = np.nonzero(f != of)[0]
        if len(bh) or len(bf):
            nbad += 1
            if nbad < 6:
                print("  row", r, "H bad cols", bh[:10], len(bh), "F bad", bf[:10], len(bf), h[bh[:3]] if len(bh) else "", oh[bh[:3]] if len(bh) else "")
    print("  bad rows", nbad)
