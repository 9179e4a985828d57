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

# the bench's device-timed step, phase by phase (events on a dedicated torch stream)
stream = torch.cuda.Stream()
torch.cuda.set_stream(stream)
sptr = stream.cuda_stream
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for rep in range(12):
    flush.fill_(rep)
    e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
    w0 = time.perf_counter()
    e[0].record(stream)
    r, _ = ctx.align_stage1_dev(dA.data_ptr(), len(A), dB.data_ptr(), len(B), *sc, k=cfg.k, sink=sink, stream=sptr)
    w1 = time.perf_counter()
    s1 = ctx.stats()
    e[1].record(stream)
    st = ctx.reverse_goal_dev(dA.data_ptr(), r.i, dB.data_ptr(), r.j, r.score, *sc, stream=sptr)
    e[2].record(stream)
    w2 = time.perf_counter()
    torch.cuda.synchronize()
    print(f"bench-like rep {rep}: stage1 {e[0].elapsed_time(e[1]):.2f} ms (wall {1e3*(w1-w0):.2f}, fill {s1['fill_ms']:.2f}, "
          f"encode {s1['encode_ms']:.2f}, reduce {s1['reduce_ms']:.2f}) reverse {e[1].elapsed_time(e[2]):.2f} ms (wall {1e3*(w2-w1):.2f})")
