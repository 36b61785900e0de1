python -c "import sys; sys.path.insert(0,'.'); from paper_conf_dac_lindlrkp19_b200.build import build; build()"
timeout 900 python -m pytest tests -m gpu -x -q -k "wl_grad or eval_tiny or eval_full or lse or det_parity or fields_sizes or high_fanout" 2>&1 | tail -3
DP_FFT=2 timeout 900 python -m pytest tests -m gpu -x -q -k "eval_tiny or eval_full or fields_tiny" 2>&1 | tail -3
B=DP_LIB_AB=paper_conf_dac_lindlrkp19_b200/lib_ab/base2.so
bash tools/ab_quick.sh "$B" "DP_FFT=0" "DP_FFT=2" "$B" "DP_FFT=0" "DP_FFT=2"
bash tools/launch_list.sh
