#!/usr/bin/env python3
"""ncu --metrics gpu__time_duration.sum --csv log -> launch list with per-kernel share:
python tools/launch_list.py launches.csv [header line]"""
import csv, sys, collections
rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10 and r[0] != "ID"]
if len(sys.argv) > 2:
    print(sys.argv[2])
tot = collections.Counter(); cnt = collections.Counter(); all_ns = 0.0
for r in rows:
    ns = float(r[14]) * (1e3 if r[13] == "us" else 1e6 if r[13] == "ms" else 1.0)
    all_ns += ns
    name = r[4][:90]
    tot[name] += ns; cnt[name] += 1
    print(f"{name:92s} {ns / 1e6:10.4f} ms")
print("# per kernel: launches, total ms, share of the listed kernel time")
for name, ns in tot.most_common():
    print(f"#  {name:90s} {cnt[name]:3d} {ns / 1e6:10.4f} ms {ns / all_ns:7.3%}")
