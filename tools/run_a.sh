set -x
timeout 600 python -m pytest tests/test_gpu_packed.py tests/test_gpu_stripes.py -x -q 2>&1 | tail -3
timeout 300 python tools/fill_bench.py C2 -1 1 --reps=3
timeout 300 python tools/fill_bench.py R10000000x1000000 1 5 6 --reps=2
