#!/bin/bash
# measurement pass after SWB_FMODE 2: gpu tests, bench line, launch list, ncu capture, variant sweep
( time timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -4 ) > gpurun_out/pytest_gpu.log 2>&1
timeout 600 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-align > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sw_fill16 -c 1 -o gpurun_out/fill16_c2 -f python tools/fill_bench.py C2 -1 --reps=1 > gpurun_out/ncu_full.log 2>&1
( timeout 600 python tools/fill_bench.py R10000000x1000000 10 5 8 1 6 0 --reps=1
  timeout 300 python tools/fill_bench.py C2 8 1 0 9 12 --reps=3 ) > gpurun_out/sweep.txt 2>&1
tail -3 gpurun_out/pytest_gpu.log; cat gpurun_out/bench_c2.json; cat gpurun_out/sweep.txt | grep -v Warn
