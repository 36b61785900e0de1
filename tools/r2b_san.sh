# round 2 (second session): compute-sanitizer over the whole ABI incl. the kept list / strays / async host path;
# the industrial-size bench (10M cells: the sort is most expensive there); ncu DRAM traffic of the walkers
rm -f gpurun_out/sanitizer_summary.txt
bash tools/sanitize.sh
python bench.py --config industrial --steps 50 --warmup 5 --skip-next --no-cpu-baseline > gpurun_out/r2b_industrial.json 2> gpurun_out/r2b_industrial.err
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:"k_(scatter_walk|gather_walk|wa_chunks|combine|row|col)" --csv \
  --log-file gpurun_out/r2b_walk_traffic.csv python bench.py --steps 6 --warmup 3 --no-cpu-baseline --e2e-steps 1 --skip-next > /dev/null 2>&1
