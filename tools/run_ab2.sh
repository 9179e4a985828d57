#!/bin/bash
bash tools/run_i32.sh
for n in i1 u8 tt; do
  export SWB_LIB=build/lib_$n.so
  echo "=== $n"
  timeout 300 python tools/fill_bench.py C2 8 --reps=3
  timeout 300 python tools/fill_bench.py R10000000x1000000 10 8 --reps=1
done 2>&1 | grep -v Warn | tee gpurun_out/ab2.txt
