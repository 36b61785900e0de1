# Round 2 (second session) final evidence on one B200: every GPU test, smoke, bench lines (bigblue4 default
# and the driver's 20/5, adaptec1, industrial), the reference arm, launch list and ncu --set full.
set -x
python -c "import sys; sys.path.insert(0,'.'); from paper_conf_dac_lindlrkp19_b200.build import build; build()"
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -5 > gpurun_out/fin_gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/fin_smoke.log 2>&1
python bench.py > gpurun_out/fin_bench_bigblue4.json 2> gpurun_out/fin_bench.err
python bench.py --steps 20 --warmup 5 > gpurun_out/fin_bench_driverlike.json 2>> gpurun_out/fin_bench.err
python bench.py --config adaptec1 --steps 500 --skip-next --no-cpu-baseline > gpurun_out/fin_bench_adaptec1.json 2>> gpurun_out/fin_bench.err
python bench.py --config industrial --steps 50 --warmup 5 --skip-next --no-cpu-baseline > gpurun_out/fin_bench_industrial.json 2>> gpurun_out/fin_bench.err
python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/fin_bench_reference.json 2>> gpurun_out/fin_bench.err
bash tools/launch_list.sh > gpurun_out/fin_launches.txt 2>&1
ncu --set full --clock-control none --import-source on \
    -k regex:"k_(wa_chunks|scatter_walk|gather_walk|row_inv_w|col_fwd_w|row_dct_w|combine)" --launch-skip 40 --launch-count 10 \
    -o gpurun_out/prof_fin python bench.py --steps 4 --warmup 4 --no-cpu-baseline --e2e-steps 1 --skip-next --no-sort-every > gpurun_out/ncu_fin.log 2>&1
python tools/ncu_table.py gpurun_out/prof_fin.ncu-rep > gpurun_out/ncu_fin_table.txt 2>&1
python tools/ncu_traffic.py gpurun_out/prof_fin.ncu-rep > gpurun_out/ncu_fin_traffic.txt 2>&1
cp profiles/ncu_wa_traffic.json gpurun_out/ncu_wa_traffic_fin.json
