# round-1 measurement pass: bench line, launch list, one full ncu capture of the fill
set -x
timeout 600 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sw_fill16 -c 1 -o gpurun_out/fill16_c2 -f python tools/fill_bench.py C2 -1 --reps=1 > gpurun_out/ncu_full.log 2>&1
timeout 900 python tools/fill_bench.py C3 -1 --reps=1
timeout 900 python tools/fill_bench.py C4 -1 --reps=1
