python -c "import sys; sys.path.insert(0,'.'); from paper_conf_dac_lindlrkp19_b200.build import build; build()"
timeout 1200 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -4
B=DP_LIB_AB=paper_conf_dac_lindlrkp19_b200/lib_ab/base.so
bash tools/ab_quick.sh "$B" "DP_FFT=0" "$B" "DP_FFT=0"
