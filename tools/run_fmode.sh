#!/bin/bash
# A/B of the packed kernel's F-chain instruction mix (SWB_FMODE builds in build/).
for m in 0 1 2; do
  export SWB_LIB=build/lib_f$m.so
  echo "=== fmode $m"
  timeout 300 python tools/fill_bench.py C2 8 1 10 --reps=3
  timeout 300 python tools/fill_bench.py C3 -1 --reps=1
  timeout 300 python tools/fill_bench.py C4 -1 --reps=1
done 2>&1 | grep -v Warning > gpurun_out/fmode.txt
for m in 1 2; do
  export SWB_LIB=build/lib_f$m.so
  echo "=== parity fmode $m"
  timeout 900 python -m pytest tests/test_gpu_packed.py tests/test_gpu_parity.py tests/test_gpu_stripes.py -x -q 2>&1 | tail -2
done >> gpurun_out/fmode.txt 2>&1
cat gpurun_out/fmode.txt
