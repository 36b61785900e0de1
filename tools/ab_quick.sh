# quick headline A/B: bench.py value + stages for each env setting given as arguments
for cfg in "$@"; do
  echo "== $cfg"; env $cfg python bench.py --steps 500 --warmup 20 --no-cpu-baseline --e2e-steps 2 2>&1 | tail -1 | grep -o '"value": [0-9.]*\|"stages_us": {[^}]*}\|"avg_launch_us_alone": [0-9.]*' | head -3
done
