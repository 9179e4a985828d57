# One C5 (32.8M x 46.9M, the paper's 33x47 MBP shape) Stage-1 run on one B200: fill time and result.
set -x
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,power.draw --format=csv
timeout 1500 python tools/fill_bench.py C5 -1 --reps=1
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,power.draw,clocks_throttle_reasons.active --format=csv
