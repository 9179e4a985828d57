"""Wall-clock breakdown of one bench step (C2) by phase."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
from paper_conf_ipps_sandesm11_b200 import Context

cfg = synth.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "C2"]
A, B = synth.make_pair(cfg)
dA, dB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
ctx = Context(0)
sc = (1, -3, 3, 2)
cnt = [0]
def sink(r, H, F):
    cnt[0] += 1
    return False
def t(f):
    torch.cuda.synchronize(); t0 = time.perf_counter(); r = f(); torch.cuda.synchronize(); return r, 1e3 * (time.perf_counter() - t0)
for rep in range(3):
    r, t_k0 = t(lambda: ctx.align_stage1_dev(dA.data_ptr(), len(A), dB.data_ptr(), len(B), *sc, k=0)[0])
    s0 = ctx.stats()
    r, t_k = t(lambda: ctx.align_stage1_dev(dA.data_ptr(), len(A), dB.data_ptr(), len(B), *sc, k=cfg.k, sink=sink)[0])
    s1 = ctx.stats()
    st, t_rev = t(lambda: ctx.reverse_goal_dev(dA.data_ptr(), r.i, dB.data_ptr(), r.j, r.score, *sc))
    s2 = ctx.stats()
    print(f"rep {rep}: stage1 k=0 {t_k0:.1f} ms (fill {s0['fill_ms']:.1f}); stage1 k={cfg.k} {t_k:.1f} ms (fill {s1['fill_ms']:.1f}, rows {s1['special_rows']}); "
          f"reverse {t_rev:.1f} ms (fill {s2['fill_ms']:.2f}, launches {s2['kernel_launches']})")
