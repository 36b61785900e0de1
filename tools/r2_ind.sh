# after the radix-16 field passes: every GPU test, smoke, industrial (2048^2) bench, bigblue4 bench, fields at 2048/4096 alone
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -4
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
python bench.py --config industrial --steps 50 --warmup 5 --skip-next --no-cpu-baseline > gpurun_out/ind_bench.json 2> gpurun_out/ind_bench.err; tail -c 600 gpurun_out/ind_bench.json
python tools/chain_times.py industrial
bash tools/ab_quick.sh DP_FFT=0
