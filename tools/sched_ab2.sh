# A/B of the WA start point (DP_SCHED): 1 = after the density map, 2 = after the placement, 3 = after the count
for rep in 1 2; do
for cfg in "DP_SCHED=1" "DP_SCHED=2" "DP_SCHED=3"; do
  echo "== $cfg"; env $cfg python bench.py --steps 500 --warmup 20 --no-cpu-baseline --e2e-steps 2 2>&1 | tail -1 | grep -o '"value": [0-9.]*\|"stages_us": {[^}]*}' | head -2
done
done
