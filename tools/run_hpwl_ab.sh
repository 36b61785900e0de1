# fused-HPWL A/B of two in-tree builds + the HPWL bit-exact tests of the candidate
DP_LIB_AB=$2 timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "hpwl or eval_tiny or virtual or one_rank" 2>&1 | tail -1
for rep in 1 2; do for lib in "$1" "$2"; do
  echo "== $lib"; DP_LIB_AB=$lib python bench.py --steps 300 --warmup 10 --no-cpu-baseline --e2e-steps 2 --skip-next 2>&1 | tail -1 | grep -o '"value": [0-9.]*\|"fused_hpwl_evals_per_s": [0-9.]*'
done; done
