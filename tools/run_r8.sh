#!/bin/bash
( timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -2 ) > gpurun_out/pytest_gpu.log 2>&1
( timeout 300 python tools/fill_bench.py C2 8 --reps=3; timeout 300 python tools/fill_bench.py R10000000x1000000 10 --reps=1; timeout 300 python tools/fill_bench.py C2 8 --reps=3 ) 2>&1 | grep GCUPS
timeout 600 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
grep -E "passed|failed" gpurun_out/pytest_gpu.log; cut -c1-200 gpurun_out/bench_c2.json
