# round-2 quick check: focused GPU parity, headline A/B (new vs DP_FFT=0), ncu launch list
set -x
python -c "import sys; sys.path.insert(0,'.'); from paper_conf_dac_lindlrkp19_b200.build import build; build()"
timeout 900 python -m pytest tests -m gpu -x -q -k "fields or transforms or density_map or density_grad or eval_tiny or eval_full or bitwise or fixed_map or virtual" 2>&1 | tail -15
bash tools/ab_quick.sh "DP_FFT=1" "DP_FFT=0" "DP_FFT=1"
bash tools/launch_list.sh
