# ncu --set full of the walkers and WA (current build), with source-line stall tables
ncu --set full --clock-control none --import-source on -k regex:"k_(wa_chunks|scatter_walk|gather_walk)" \
    --launch-skip 30 --launch-count 6 -o gpurun_out/prof3 python bench.py --steps 4 --warmup 4 \
    --no-cpu-baseline --e2e-steps 1 --skip-next > gpurun_out/ncu3.log 2>&1
python tools/ncu_table.py gpurun_out/prof3.ncu-rep > gpurun_out/ncu3_table.txt 2>&1
python tools/ncu_lines.py gpurun_out/prof3.ncu-rep k_scatter_walk 30 > gpurun_out/ncu3_scatter_lines.txt 2>&1
python tools/ncu_lines.py gpurun_out/prof3.ncu-rep k_gather_walk 30 > gpurun_out/ncu3_gather_lines.txt 2>&1
python tools/ncu_sass.py gpurun_out/prof3.ncu-rep k_scatter_walk 25 > gpurun_out/ncu3_scatter_sass.txt 2>&1
