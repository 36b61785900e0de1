python -c "import sys; sys.path.insert(0,'.'); from paper_conf_dac_lindlrkp19_b200.build import build; build()"
timeout 900 python -m pytest tests -m gpu -x -q -k "wl_grad or eval_tiny or eval_full or lse or det or high_fanout or gp or fixed" 2>&1 | tail -3
B=DP_LIB_AB=paper_conf_dac_lindlrkp19_b200/lib_ab/base2.so
bash tools/ab_quick.sh "$B" "DP_X=0" "$B" "DP_X=0"
bash tools/launch_list.sh
