python -c "import sys; sys.path.insert(0,'.'); from paper_conf_dac_lindlrkp19_b200.build import build; build()"
timeout 1500 python -m pytest tests -m gpu -x -q -k "regions or fixed or gp" 2>&1 | tail -3
