set -x
ncu --set full --clock-control none --import-source on -k regex:"k_(combine|place|count|col_fields|scatter_walk|gather_walk|row_inv|row_dct|scan|wa_big|scatter_large|gather_large|finalize)" --launch-skip 30 --launch-count 14 -o gpurun_out/prof_all python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/ncu_all.log 2>&1
ls -la gpurun_out
