"""Band timeline of the last Stage-2 partition (SWB_DEBUG_TIMES=1): where does a
partition's time go?  python tools/stage2_bands.py [m] [k]"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["SWB_DEBUG_TIMES"] = "1"
import numpy as np
import synth
from paper_conf_ipps_sandesm11_b200 import Context
from tools.fill_bench import band_times

m = int(sys.argv[1]) if len(sys.argv) > 1 else 400000
k = int(sys.argv[2]) if len(sys.argv) > 2 else 65536
A, B = synth.random_pair(3, m, m, plant_len=m, s=5e-5, g=3e-5, mu=10)
ctx = Context(0)
r, _ = ctx.align_stage1(A, B, 1, -3, 3, 2, k=k)
for rep in range(2):
    t0 = time.perf_counter()
    L = ctx.stage2(A, B, 1, -3, 3, 2, k=k, end=r)
    t1 = time.perf_counter()
    print(f"stage2 {1e3*(t1-t0):.1f} ms |L|={len(L)} stats={ctx.stats()}")
a = band_times(ctx)  # the last partition (rows 0..k): columns 0 start, 1 first tile, 15 end (us)
import ctypes
buf = (ctypes.c_uint64 * (80 * 40000))()
nn = ctx._lib.swb_debug_times(ctx._h, buf, len(buf))
raw = np.frombuffer(buf, dtype=np.uint64, count=nn).reshape(-1, 80)
for b in list(range(0, 20)) + [40, 80, 147]:
    if b < len(a):
        print(f"band {b:4d}: first-tile {a[b,1]:9.1f} q1 {a[b,2]:9.1f} q2 {a[b,3]:9.1f} q3 {a[b,4]:9.1f} end {a[b,15]:9.1f}  "
              f"waits {raw[b,7]} spins {raw[b,6]} wait_ms {raw[b,5]/1e6:.2f} replays {raw[b,9]}")
