python -c "import sys; sys.path.insert(0,'.'); from paper_conf_dac_lindlrkp19_b200.build import build; build()"
W=DP_LIB_AB=paper_conf_dac_lindlrkp19_b200/lib_ab/wa512.so
DP_LIB_AB=paper_conf_dac_lindlrkp19_b200/lib_ab/wa512.so timeout 900 python -m pytest tests -m gpu -x -q -k "wl_grad or eval_tiny or eval_full or high_fanout or virtual or det_bitwise" 2>&1 | tail -2
bash tools/ab_quick.sh "DP_X=0" "DP_T2B_WARPS=2" "$W" "$W DP_T2B_WARPS=2" "DP_X=0" "$W"
DP_LIB_AB=paper_conf_dac_lindlrkp19_b200/lib_ab/wa512.so python tools/chain_times.py
