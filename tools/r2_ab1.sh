python -c "import sys; sys.path.insert(0,'.'); from paper_conf_dac_lindlrkp19_b200.build import build; build()"
timeout 600 python -m pytest tests -m gpu -x -q -k "density or fixed_map or eval_tiny or virtual or bitwise" 2>&1 | tail -2
B=DP_LIB_AB=paper_conf_dac_lindlrkp19_b200/lib_ab/base.so
bash tools/ab_quick.sh "$B" "DP_FFT=0" "DP_FFT=2" "DP_WALK_CTAS=2" "$B" "DP_FFT=0" "DP_FFT=2" "DP_WALK_CTAS=2"
bash tools/launch_list.sh
