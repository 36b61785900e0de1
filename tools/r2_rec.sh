# 16-byte density records: GPU parity (all non-slow GPU tests + full-size eval / sweep), headline A/B
python -c "import sys; sys.path.insert(0,'.'); from paper_conf_dac_lindlrkp19_b200.build import build; build()"
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -4
bash tools/ab_quick.sh "DP_WALK_CTAS=9" "DP_WALK_CTAS=2" "DP_WALK_CTAS=9" "DP_WALK_CTAS=2"
bash tools/launch_list.sh
