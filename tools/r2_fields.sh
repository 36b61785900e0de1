# fields A/B: parity of the field passes, headline new vs DP_FFT=0, launch list
python -c "import sys; sys.path.insert(0,'.'); from paper_conf_dac_lindlrkp19_b200.build import build; build()"
timeout 600 python -m pytest tests -m gpu -x -q -k "fields or eval_tiny or transforms" 2>&1 | tail -3
bash tools/ab_quick.sh "DP_FFT=1" "DP_FFT=0"
bash tools/launch_list.sh
ncu --set full --clock-control none --import-source on -k regex:"k_p[123]" --launch-skip 30 --launch-count 3 \
    -o gpurun_out/prof_fields python bench.py --steps 4 --warmup 4 --no-cpu-baseline --e2e-steps 1 --skip-next > gpurun_out/ncu_fields.log 2>&1
