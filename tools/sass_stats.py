#!/usr/bin/env python3
"""Per-function SASS opcode histogram, and per-loop histograms (backward branches)
for a cubin/so: python tools/sass_stats.py lib.so [function-substring]."""
import re, subprocess, sys, collections

def functions(path):
    out = subprocess.run(["cuobjdump", "-sass", path], capture_output=True, text=True).stdout
    cur, lines = None, []
    for ln in out.splitlines():
        m = re.match(r"\s*Function : (\S+)", ln)
        if m:
            if cur: yield cur, lines
            cur, lines = m.group(1), []
        elif cur:
            lines.append(ln)
    if cur: yield cur, lines

INS = re.compile(r"/\*([0-9a-f]{4,})\*/\s+(@!?U?P\w+\s+)?([A-Z][A-Z0-9_.]*)\s*([^;]*);")

def parse(lines):
    ins = []
    for ln in lines:
        m = INS.search(ln)
        if m:
            ins.append((int(m.group(1), 16), m.group(3), m.group(4)))
    return ins

def main():
    path = sys.argv[1]
    pat = sys.argv[2] if len(sys.argv) > 2 else ""
    for name, lines in functions(path):
        if pat not in name: continue
        ins = parse(lines)
        h = collections.Counter(op.split(".")[0] for _, op, _ in ins)
        print(f"== {name}: {len(ins)} instrs; LDL={h['LDL']} STL={h['STL']}")
        addr = {a: i for i, (a, _, _) in enumerate(ins)}
        loops = []
        for i, (a, op, args) in enumerate(ins):
            if op.startswith("BRA"):
                m = re.search(r"0x([0-9a-f]+)", args)
                if m:
                    tgt = int(m.group(1), 16)
                    if tgt < a and tgt in addr:
                        loops.append((addr[tgt], i))
        for s, e in loops:
            body = ins[s:e + 1]
            hh = collections.Counter(op.split(".")[0] for _, op, _ in body)
            if hh["VIADDMNMX"] >= 16:
                print(f"  loop [{s}:{e}] {len(body)} instrs: " + ", ".join(f"{k}={v}" for k, v in hh.most_common(14)))

main()
