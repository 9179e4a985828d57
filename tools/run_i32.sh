#!/bin/bash
# int32 kernel A/B (H form vs D form, runtime vs patched immediates) and its parity tests
for n in old i0 i1; do
  export SWB_LIB=build/lib_$n.so
  for p in 1 0; do
    [ $n = old ] && [ $p = 0 ] && continue
    echo "=== $n SWB_PATCH=$p"
    SWB_PATCH=$p timeout 300 python tools/rev_bench.py 2000000
  done
done 2>&1 | grep -v Warn > gpurun_out/i32_ab.txt
export SWB_LIB=build/lib_i1.so
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_variants.py tests/test_gpu_stage2.py tests/test_gpu_align.py tests/test_gpu_stripes.py -x -q 2>&1 | tail -3 >> gpurun_out/i32_ab.txt
cat gpurun_out/i32_ab.txt
