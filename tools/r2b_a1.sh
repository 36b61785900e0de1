# adaptec1: reuse on / off with the two graph variants (bench walk + GP)
for v in "DP_REUSE_SORT=0" "DP_REUSE_SORT=1" "DP_REUSE_SORT=0" "DP_REUSE_SORT=1"; do
  echo "== $v"; env $v python bench.py --config adaptec1 --steps 500 --warmup 20 --no-cpu-baseline --e2e-steps 2 --skip-next --no-sort-every 2>&1 | tail -1 | grep -o '"value": [0-9.]*' | head -1
  env $v python tools/gp_prof.py adaptec1 600
done
