# ncu full + source of the top kernels (one launch each) and the 2048^2 fields A/B
python -c "import sys; sys.path.insert(0,'.'); from paper_conf_dac_lindlrkp19_b200.build import build; build()"
ncu --set full --clock-control none --import-source on \
    -k regex:"k_(wa_chunks|place|scatter_walk|gather_walk|count)" --launch-skip 20 --launch-count 5 \
    -o gpurun_out/prof_top python bench.py --steps 4 --warmup 4 --no-cpu-baseline --e2e-steps 1 --skip-next > gpurun_out/ncu_top.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "fields_sizes or bin_sweep or gp_one_step or gp_first" 2>&1 | tail -5
for f in 1 0; do DP_FFT=$f python bench.py --config industrial --steps 50 --warmup 5 --no-cpu-baseline --e2e-steps 1 --skip-next 2>&1 | tail -1 | grep -o '"value": [0-9.]*\|"stages_us": {[^}]*}'; done
