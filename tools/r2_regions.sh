python -c "import sys; sys.path.insert(0,'.'); from paper_conf_dac_lindlrkp19_b200.build import build; build()"
timeout 900 python -m pytest tests -m gpu -x -q -k "regions or fixed or gp_overflow or recapture" 2>&1 | tail -5
mkdir -p gpurun_out
bash tools/sanitize.sh
cat gpurun_out/sanitizer_summary.txt
