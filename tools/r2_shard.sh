python -c "import sys; sys.path.insert(0,'.'); from paper_conf_dac_lindlrkp19_b200.build import build; build()"
timeout 900 python -m pytest tests -m gpu -x -q -k "sharded or one_rank or virtual or det_gradient or fields_sizes" 2>&1 | tail -8
