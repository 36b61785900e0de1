for A in 0 1 2 3 4; do
  DP_ABLATE_PLACE=$A ncu --metrics gpu__time_duration.sum --clock-control none -k regex:k_place -s 5 -c 3 --csv --log-file gpurun_out/abl_$A.csv python bench.py --steps 4 --warmup 4 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1
  echo "ablate=$A"; grep k_place gpurun_out/abl_$A.csv | awk -F'","' '{print $NF}' | tr -d '"' | head -3
done
