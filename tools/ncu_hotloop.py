#!/usr/bin/env python3
"""Per-SASS stall samples of an ncu source page (csv from
`ncu -i rep --page source --csv --print-source sass`): totals by reason, the
hottest instructions, and optionally one address range.
python tools/ncu_hotloop.py src.csv [lo_off hi_off]"""
import csv, sys, collections
rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]; data = rows[2:]
ix = {h: i for i, h in enumerate(hdr)}
cols = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
recs = []
for r in data:
    try:
        a = int(r[0], 16)
    except ValueError:
        continue
    s = int(r[ix["# Samples"]] or 0)
    st = {c: int(r[ix[c]] or 0) for c in cols}
    recs.append((a, r[1].strip(), s, st, int(r[ix["Instructions Executed"]] or 0)))
base = recs[0][0]
allS = sum(x[2] for x in recs)
tot = collections.Counter({c: sum(x[3][c] for x in recs) for c in cols})
print("total samples", allS)
print("by reason:", ", ".join(f"{c[6:]}={v/allS:.3f}" for c, v in tot.most_common(10)))
print("top instructions:")
for a, src, s, st, ex in sorted(recs, key=lambda x: -x[2])[:25]:
    top = ", ".join(f"{c[6:]}={v}" for c, v in sorted(st.items(), key=lambda kv: -kv[1])[:3] if v)
    print(f"  {a-base:6x} {s:7d} {src[:60]:60s} {top}")
if len(sys.argv) > 3:
    lo, hi = int(sys.argv[2], 16), int(sys.argv[3], 16)
    sel = [x for x in recs if lo <= x[0] - base <= hi]
    S = sum(x[2] for x in sel) or 1
    print(f"region {lo:x}-{hi:x}: {S} samples ({S/allS:.3f}), {len(sel)} instrs")
    c2 = collections.Counter()
    for x in sel:
        for c, v in x[3].items(): c2[c] += v
    print("  by reason:", ", ".join(f"{c[6:]}={v/S:.3f}" for c, v in c2.most_common(8)))
    for a, src, s, st, ex in sel:
        top = ", ".join(f"{c[6:]}={v}" for c, v in sorted(st.items(), key=lambda kv: -kv[1])[:2] if v)
        print(f"  {a-base:6x} {s:6d} {src[:58]:58s} {top}")
