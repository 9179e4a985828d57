# Which nvidia-smi clock query perturbs a running step (host-driven special-row loop)?
for q in "clocks.sm,clocks.max.sm,clocks_event_reasons.active" "clocks.sm,clocks.max.sm,power.draw" "clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap"; do
  echo "== $q"
  ( time -p nvidia-smi -i 0 --query-gpu=$q --format=csv,noheader,nounits ) 2>&1 | tr '\n' ' '; echo
  nvidia-smi -i 0 --query-gpu=$q --format=csv,noheader,nounits -lms 200 > /dev/null &
  P=$!
  timeout 100 python tools/step_breakdown.py 2>&1 | grep bench-like | awk '{print $5}' | tr '\n' ' '; echo
  kill $P
done
