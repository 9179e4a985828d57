#!/bin/bash
# Variant sweep on one workload: tools/sweep.sh <workload> <variants...>
wl=$1; shift
for v in "$@"; do
  SWB_VARIANT=$v timeout 600 python bench.py --workload $wl --steps 3 --warmup 2 --no-cpu-baseline --no-e2e > gpurun_out/sweep_${wl}_v$v.json 2>gpurun_out/sweep_${wl}_v$v.err
  python -c "import json;d=json.load(open('gpurun_out/sweep_${wl}_v$v.json'));print('$wl', $v, d['value'], 'fill_ms', d['roofline']['fill_ms'], 'frac', d['roofline']['frac'], d['config']['kernel'], d['result'], 'replays', d['replays_per_step'], d['clocks'])" || tail -5 gpurun_out/sweep_${wl}_v$v.err
done
