python -c "import sys; sys.path.insert(0,'.'); from paper_conf_dac_lindlrkp19_b200.build import build; build()"
R=DP_LIB_AB=paper_conf_dac_lindlrkp19_b200/lib_ab/rec16.so
DP_LIB_AB=paper_conf_dac_lindlrkp19_b200/lib_ab/rec16.so timeout 600 python -m pytest tests -m gpu -x -q -k "density or eval_tiny or fixed_map or bitwise" 2>&1 | tail -2
bash tools/ab_quick.sh "DP_X=0" "$R" "$R DP_WALK_CTAS=2" "$R DP_WA_CHUNK=2048" "$R DP_WA_CHUNK=2048 DP_WALK_CTAS=2" "DP_WA_CHUNK=2048 DP_WALK_CTAS=1" "DP_X=0" "$R DP_WA_CHUNK=2048"
timeout 1500 python -m pytest tests -m "gpu and slow" -x -q -k "initial_full or gamma_lambda or overflow_with_fixed or recaptures" 2>&1 | tail -3
