#!/bin/bash
# patched-immediate packed kernel: parity, A/B timing against the register-operand kernel
timeout 900 python -m pytest tests/test_gpu_packed.py -x -q 2>&1 | tail -3 > gpurun_out/patch_tests.txt
for p in 1 0; do
  export SWB_PATCH=$p
  echo "=== SWB_PATCH=$p"
  timeout 300 python tools/fill_bench.py C2 8 -1 --reps=3
  timeout 300 python tools/fill_bench.py R10000000x1000000 10 8 1 5 6 --reps=1
done 2>&1 | grep -v Warn > gpurun_out/patch_ab.txt
cat gpurun_out/patch_tests.txt gpurun_out/patch_ab.txt
