# Full ncu sections for one launch of each top kernel (run under gpurun; one GPU).
ncu --set full --clock-control none --import-source on \
    -k regex:"k_(wa_chunks|place|col_fields|scatter_walk|gather_walk|combine|count|wa_big|row_inv|row_dct)" \
    --launch-skip 40 --launch-count 12 -o gpurun_out/prof_top python bench.py --steps 4 --warmup 4 \
    --no-cpu-baseline --e2e-steps 1 --skip-next > gpurun_out/ncu_top.log 2>&1
