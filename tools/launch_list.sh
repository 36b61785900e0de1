# ncu launch list (per-kernel duration, cold-cache, serialised) of a short bench run -> gpurun_out/launches.txt
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_" --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 1 --skip-next --no-sort-every > /dev/null 2>&1
python tools/launches.py gpurun_out/launches.csv > gpurun_out/launches.txt 2>&1
grep -v "wa_chunks<1>\|wa_chunks<2>" gpurun_out/launches.txt
