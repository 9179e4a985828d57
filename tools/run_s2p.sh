#!/bin/bash
timeout 900 python -m pytest tests/test_gpu_stage2.py tests/test_gpu_align.py -x -q 2>&1 | tail -2
for v in 1 0; do echo "== SWB_S2PACKED=$v"; SWB_S2PACKED=$v REV=0 timeout 900 python tools/stage2_bench.py C3 C4 2>&1 | grep -v Warn | tail -2; done
