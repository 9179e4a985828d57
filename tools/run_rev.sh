#!/bin/bash
( time timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -4 ) > gpurun_out/pytest_gpu.log 2>&1
timeout 300 python tools/rev_bench.py 2000000 > gpurun_out/rev_bench.txt 2>&1
timeout 600 python bench.py --workload C3 --steps 3 --warmup 3 --no-align --no-cpu-baseline > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err
grep -E "passed|failed" gpurun_out/pytest_gpu.log; grep -A1 m= gpurun_out/rev_bench.txt; cat gpurun_out/bench_c3.json
