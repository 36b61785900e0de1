python -c "import sys; sys.path.insert(0,'.'); from paper_conf_dac_lindlrkp19_b200.build import build; build()"
DP_MAP=direct timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "eval_tiny or eval_full or initial_full or density_grad" 2>&1 | tail -3
bash tools/ab_quick.sh "DP_X=0" "DP_MAP=direct" "DP_MAP=direct DP_SCHED=0" "DP_X=0" "DP_MAP=direct"
DP_MAP=direct python tools/chain_times.py
python tools/chain_times.py
DP_MAP=direct bash tools/launch_list.sh
