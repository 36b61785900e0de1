python -c "import sys; sys.path.insert(0,'.'); from paper_conf_dac_lindlrkp19_b200.build import build; build()"
timeout 1500 python -m pytest tests -m gpu -x -q -k "density or fixed or eval or bitwise or virtual or regions or bin_sweep or initial_full" 2>&1 | tail -3
B=DP_LIB_AB=paper_conf_dac_lindlrkp19_b200/lib_ab/base3.so
bash tools/ab_quick.sh "$B" "DP_X=0" "$B" "DP_X=0"
bash tools/launch_list.sh
