# A/B of alternative in-tree builds (paper_conf_dac_lindlrkp19_b200/lib_ab/*.so): parity subset, then headline
for lib in "$@"; do
  DP_LIB_AB=$lib timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "density or eval_tiny or virtual" 2>&1 | tail -1
done
args=()
for rep in 1 2; do for lib in "$@"; do args+=("DP_LIB_AB=$lib"); done; done
bash tools/ab_quick.sh "${args[@]}"
