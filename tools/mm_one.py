import os, sys, time
sys.path.insert(0, os.getcwd())
import synth
from paper_conf_ipps_sandesm11_b200 import Context
N = int(sys.argv[1])
A, B = synth.random_pair(5, N, N, plant_len=N, s=0.01, g=0.002)
with Context(0) as ctx:
    for _ in range(2):
        t0 = time.perf_counter(); r = ctx.align(A, B, 1, -3, 3, 2, k=0); t1 = time.perf_counter()
        print(N, r['score'], r['partitions'], r['mm_levels'], f"{1e3*(t1-t0):.1f} ms", r['ms'], flush=True)
