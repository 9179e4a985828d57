#!/usr/bin/env python3
"""Summarise an ncu report (raw page) for profiles/: python tools/ncu_summary.py rep.ncu-rep [cells]"""
import csv, io, subprocess, sys
rep = sys.argv[1]
cells = float(sys.argv[2]) if len(sys.argv) > 2 else None
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr, units, vals = rows[0], rows[1], rows[2]
d = {h: (v, u) for h, u, v in zip(hdr, units, vals)}
keys = ["Kernel Name", "gpu__time_duration.sum", "launch__grid_size", "launch__block_size", "launch__registers_per_thread",
        "dram__bytes_read.sum", "dram__bytes_write.sum", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active", "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active", "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.per_cycle_active", "smsp__inst_executed.sum", "sm__cycles_active.avg",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "gpc__cycles_elapsed.max", "sm__cycles_elapsed.avg.per_second"]
for k in keys:
    if k in d:
        print(f"{k:65s} {d[k][0]:>22s} {d[k][1]}")
st = sorted(((h, float(v or 0)) for h, (v, u) in d.items() if h.startswith("smsp__average_warps_issue_stalled") and h.endswith("per_issue_active.ratio")), key=lambda x: -x[1])[:10]
print("-- top stall reasons (warps per issue)")
for h, v in st:
    print(f"  {h.replace('smsp__average_warps_issue_stalled_', '').replace('_per_issue_active.ratio', ''):40s} {v:.3f}")
if cells:
    inst = float(d["smsp__inst_executed.sum"][0])
    print(f"-- warp-instructions x 32 / cell = {inst * 32 / cells:.3f}")
    print(f"-- dram bytes / cell = {(float(d['dram__bytes_read.sum'][0]) * (1e6 if d['dram__bytes_read.sum'][1]=='Mbyte' else 1) + float(d['dram__bytes_write.sum'][0]) * (1e6 if d['dram__bytes_write.sum'][1]=='Mbyte' else 1)) / cells:.5f}")
