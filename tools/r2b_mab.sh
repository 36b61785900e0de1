# walker margin A/B (m = 0, 2, 4) with the small scatter CTA: headline + GP from the P:153 start
python -m pytest tests -m gpu -q -x 2>&1 | tail -3 > gpurun_out/mab_tests.log
L=paper_conf_dac_lindlrkp19_b200/lib_ab
for v in "DP_LIB_AB=$L/m0.so" "DP_LIB_AB=$L/m2.so" "DP_MARGIN_DEFAULT=4" "DP_REUSE_SORT=0"; do
  echo "== $v"; env $v python tools/gp_prof.py bigblue4 20; env $v python tools/gp_prof.py bigblue4 600; env $v python tools/gp_prof.py adaptec1 600
  env $v python bench.py --steps 300 --warmup 20 --no-cpu-baseline --e2e-steps 2 --skip-next 2>&1 | tail -1 | grep -o '"value": [0-9.]*\|"hot_back_to_back_evals_per_s": [0-9.]*\|"stages_us": {[^}]*}' | head -3
done
