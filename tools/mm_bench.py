#!/usr/bin/env python3
"""Full alignment of a whole-length synthetic pair (one Stage-2 partition):
python tools/mm_bench.py N [k] -- times sw_align and its Myers-Miller levels."""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402
from paper_conf_ipps_sandesm11_b200 import Context  # noqa: E402

N = int(sys.argv[1]) if len(sys.argv) > 1 else 20000
k = int(sys.argv[2]) if len(sys.argv) > 2 else 0
A, B = synth.random_pair(5, N, N, plant_len=N, s=0.01, g=0.002)
with Context(0) as ctx:
    t0 = time.perf_counter()
    r = ctx.align(A, B, 1, -3, 3, 2, k=k)
    t1 = time.perf_counter()
    print(f"N={N} k={k} score={r['score']} partitions={r['partitions']} levels={r['mm_levels']} "
          f"wall {1e3*(t1-t0):.1f} ms", r["ms"])
