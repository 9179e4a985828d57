#!/bin/bash
# C5 Stage 1 (paper's 33x47 MBP shape) with the patched packed kernel, and a C4 bench line
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/c5.txt
timeout 1500 python tools/fill_bench.py C5 -1 --reps=1 2>&1 | grep -v Warn >> gpurun_out/c5.txt
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,power.draw,clocks_throttle_reasons.active --format=csv >> gpurun_out/c5.txt
timeout 900 python bench.py --workload C4 --steps 3 --warmup 3 --no-align > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err
cat gpurun_out/c5.txt gpurun_out/bench_c4.json
