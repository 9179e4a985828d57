python tools/mm_bench.py 20000
SWB_MM_CTA_ROWS=100000000 python tools/mm_bench.py 20000
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sw_mm_split_cta -c 1 -o gpurun_out/mm_cta -f python tools/mm_bench.py 20000 > gpurun_out/ncu_mm.log 2>&1
