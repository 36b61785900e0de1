# A/B of env-switch configurations on the bench headline (run under gpurun, one GPU).
# usage: bash tools/ab.sh "ENV=a ENV2=b" "ENV=c" ...
for cfg in "$@"; do
  echo "== $cfg"
  env $cfg python bench.py --steps 500 --warmup 10 --no-cpu-baseline --e2e-steps 2 2>&1 | tail -1 | grep -o '"value": [0-9.]*\|"stages_us": {[^}]*}' | head -2
done
