set -x
timeout 900 python -m pytest tests/test_gpu_align.py tests/test_gpu_stage2.py -x -q 2>&1 | tail -3
timeout 900 python tools/align_bench.py C1 C2 C4 C3
