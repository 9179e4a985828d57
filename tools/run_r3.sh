#!/bin/bash
# measurement pass: gpu tests, bench line, launch list, ncu capture of the C2 fill, C3/C4 fills
( time timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -4 ) > gpurun_out/pytest_gpu.log 2>&1
timeout 600 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-align > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sw_fill16 -c 1 -o gpurun_out/fill16p_c2 -f python tools/fill_bench.py C2 -1 --reps=1 > gpurun_out/ncu_full.log 2>&1
( timeout 300 python tools/fill_bench.py C3 -1 --reps=1
  timeout 300 python tools/fill_bench.py C4 -1 --reps=1 ) 2>&1 | grep -v Warn > gpurun_out/fills.txt
tail -3 gpurun_out/pytest_gpu.log; cat gpurun_out/bench_c2.json; cat gpurun_out/fills.txt
