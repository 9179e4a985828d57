"""Stage 2 (crosspoints by goal-based matching) vs the plain reverse pass on a
workload: python tools/stage2_bench.py C3 [C4 ...]"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
from paper_conf_ipps_sandesm11_b200 import Context

SC = (1, -3, 3, 2)
ctx = Context(0)
for name in sys.argv[1:]:
    cfg = synth.CONFIGS[name]
    A, B = synth.make_pair(cfg)
    dA, dB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
    m, n = len(A), len(B)
    t0 = time.perf_counter()
    r, _ = ctx.align_stage1_dev(dA.data_ptr(), m, dB.data_ptr(), n, *SC, k=cfg.k, sink=lambda *a: False)
    t1 = time.perf_counter()
    L = ctx.stage2_dev(dA.data_ptr(), m, dB.data_ptr(), n, *SC, k=cfg.k, end=r)
    torch.cuda.synchronize()
    t2 = time.perf_counter()
    st2 = ctx.stats()
    gaps = sum(1 for c in L if c[3] == 2)
    print(f"{name}: stage1 {1e3*(t1-t0):.1f} ms best={r.astuple()} | stage2 {1e3*(t2-t1):.1f} ms, |L_2|={len(L)} "
          f"({gaps} gap crosspoints), fill {st2['fill_ms']:.1f} ms in {st2['kernel_launches']} launches, start={L[0]}", flush=True)
    if len(sys.argv) > 1 and os.environ.get("REV", "1") == "1":
        t3 = time.perf_counter()
        s = ctx.reverse_goal_dev(dA.data_ptr(), r.i, dB.data_ptr(), r.j, r.score, *SC)
        t4 = time.perf_counter()
        print(f"{name}: reverse pass {1e3*(t4-t3):.1f} ms start={s.astuple()}", flush=True)
