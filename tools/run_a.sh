set -x
timeout 900 python -m pytest tests/test_gpu_packed.py -x -q 2>&1 | tail -3
timeout 300 python tools/fill_bench.py C2 8 12 --reps=3
timeout 300 python tools/fill_bench.py R10000000x1000000 12 --reps=1
