for cfg in "DP_SCHED=0 DP_PRIO=0" "DP_SCHED=0 DP_PRIO=1" "DP_SCHED=1 DP_PRIO=0" "DP_SCHED=1 DP_PRIO=1" "DP_SERIAL=1"; do
  echo "== $cfg"; env $cfg python bench.py --steps 200 --warmup 10 --no-cpu-baseline --e2e-steps 2 2>&1 | tail -1 | grep -o '"value": [0-9.]*\|"stages_us": {[^}]*}' | head -2
done
