# quick headline A/B: bench.py value (L2-cold), hot back-to-back value and stages for each env setting given as arguments
for cfg in "$@"; do
  echo "== $cfg"; env $cfg python bench.py --steps 300 --warmup 20 --no-cpu-baseline --e2e-steps 2 --skip-next 2>&1 | tail -1 | grep -o '"value": [0-9.]*\|"hot_back_to_back_evals_per_s": [0-9.]*\|"stages_us": {[^}]*}\|"avg_launch_us_alone": [0-9.]*' | head -4
done
