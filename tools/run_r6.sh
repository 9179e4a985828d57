#!/bin/bash
( time timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -4 ) > gpurun_out/pytest_gpu.log 2>&1
for p in 1 0; do SWB_PATCH=$p timeout 300 python tools/fill_bench.py C2 8 --reps=3; SWB_PATCH=$p timeout 300 python tools/fill_bench.py R10000000x1000000 10 --reps=1; done 2>&1 | grep -v Warn > gpurun_out/r6_fill.txt
timeout 600 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
grep -E "passed|failed" gpurun_out/pytest_gpu.log; cat gpurun_out/r6_fill.txt; cut -c1-300 gpurun_out/bench_c2.json
