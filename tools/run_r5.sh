#!/bin/bash
( time timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -4 ) > gpurun_out/pytest_gpu.log 2>&1
timeout 600 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
timeout 300 python tools/rev_bench.py 2000000 > gpurun_out/rev_bench.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
grep -E "passed|failed" gpurun_out/pytest_gpu.log; tail -1 gpurun_out/smoke.log | cut -c1-80; grep -A1 m= gpurun_out/rev_bench.txt; cat gpurun_out/bench_c2.json
