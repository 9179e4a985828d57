import os, sys
sys.path.insert(0, os.getcwd())
os.environ["SWB_DEBUG_TIMES"] = "1"
import synth
from paper_conf_ipps_sandesm11_b200 import Context
from tools.fill_bench import band_times
ctx = Context(0)
ctx.set_kernel(1, False)
for (m, n) in [(69632, 65536), (69632, 536165)]:
    A, B = synth.random_pair(3, m, n, plant_len=60000, s=5e-5, g=3e-5, mu=10)
    for rep in range(2):
        r, _ = ctx.align_stage1(A, B, 1, -3, 3, 2, k=0)
    st = ctx.stats()
    a = band_times(ctx)
    import ctypes, numpy as np
    buf = (ctypes.c_uint64 * (80 * 40000))()
    nn = ctx._lib.swb_debug_times(ctx._h, buf, len(buf))
    raw = np.frombuffer(buf, dtype=np.uint64, count=nn).reshape(-1, 80)
    print(m, n, "fill", st["fill_ms"], "grid", st["grid"])
    for b in range(min(17, len(a))):
        print(f"  band {b:3d}: first-tile {a[b,1]:9.1f} q1 {a[b,2]:9.1f} q2 {a[b,3]:9.1f} q3 {a[b,4]:9.1f} end {a[b,15]:9.1f}  waits {raw[b,7]} spins {raw[b,6]} wait_ms {raw[b,5]/1e6:.2f}")
