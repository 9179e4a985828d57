#!/usr/bin/env python3
"""Time the int32 kernel: Stage-1 fill with the packed kernel off, and the
reverse pass (GLOBAL mode) of a whole-length alignment.
python tools/rev_bench.py [m] [variant]"""
import os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa
import synth  # noqa
from paper_conf_ipps_sandesm11_b200 import Context  # noqa

m = int(sys.argv[1]) if len(sys.argv) > 1 else 2000000
A, B = synth.random_pair(5, m, m, plant_len=m, s=0.01, g=0.001)  # whole-length homology
dA, dB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
ctx = Context(0)
ctx.set_kernel(1, False)  # int32, default geometry
for rep in range(2):
    r, _ = ctx.align_stage1_dev(dA.data_ptr(), len(A), dB.data_ptr(), len(B), 1, -3, 3, 2, k=0)
    st1 = ctx.stats()
    s = ctx.reverse_goal(A, r.i, B, r.j, r.score, 1, -3, 3, 2)
    st2 = ctx.stats()
print(f"m={m} best={r.astuple()} start={s.astuple()} int32 stage1 fill {st1['fill_ms']:.1f} ms "
      f"({len(A) * len(B) / st1['fill_ms'] / 1e6:.0f} GCUPS, patched={st1['patched']}); reverse fill {st2['fill_ms']:.1f} ms "
      f"({r.i * r.j / st2['fill_ms'] / 1e6:.0f} GCUPS, patched={st2['patched']})")
ctx.set_kernel(-1, True)  # automatic: the packed kernel in global mode
for rep in range(2):
    s = ctx.reverse_goal(A, r.i, B, r.j, r.score, 1, -3, 3, 2)
    st3 = ctx.stats()
print(f"  packed reverse fill {st3['fill_ms']:.1f} ms ({r.i * r.j / st3['fill_ms'] / 1e6:.0f} GCUPS, alpha={st3['alpha']}, "
      f"patched={st3['patched']}) start={s.astuple()}")
ctx.close()
