# clumped placement (P:153 start, GP trajectory): HEAD build vs this build with / without sort reuse
for v in "DP_LIB_AB=paper_conf_dac_lindlrkp19_b200/lib_ab/head.so" "DP_REUSE_SORT=0" "DP_REUSE_SORT=1"; do
  echo "== $v"
  env $v python tools/gp_prof.py bigblue4 20
  env $v python tools/gp_prof.py bigblue4 600
  env $v python bench.py --dist initial --steps 200 --warmup 5 --skip-next --no-cpu-baseline --e2e-steps 1 | grep -o '"value": [0-9.]*\|"stages_us": {[^}]*}'
done
for v in "DP_LIB_AB=paper_conf_dac_lindlrkp19_b200/lib_ab/head.so" "DP_REUSE_SORT=0"; do
  n=$(echo $v | tr -c 'A-Za-z0-9\n' _)
  env $v ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_" --csv --log-file gpurun_out/gp_launch_$n.csv python tools/gp_prof.py bigblue4 20 > /dev/null 2>&1
  echo "== launches $v"; python tools/launches.py gpurun_out/gp_launch_$n.csv | head -24
done
