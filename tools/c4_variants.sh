#!/bin/bash
# Stage-1 fill time of C4 per geometry (-1 = the library's automatic choice, with its tail segment)
cd "$(dirname "$0")/.."
timeout 300 python tools/fill_bench.py C4 -1 --reps=1 2>&1 | tail -1
for v in 10 14 15 16 17; do timeout 300 python tools/fill_bench.py C4 $v --reps=1 2>&1 | tail -1; done
for t in 1 14 9; do echo "tail variant $((t-1)):"; SWB_TAIL=$t timeout 300 python tools/fill_bench.py C4 10 --reps=1 2>&1 | tail -1; done
