python -c "import sys; sys.path.insert(0,'.'); from paper_conf_dac_lindlrkp19_b200.build import build; build()"
DP_GRAPH=0 DP_WALK_SYNC=1 timeout 1500 compute-sanitizer --tool racecheck --racecheck-report all --print-limit 50 \
   python tools/sanitize_run.py > gpurun_out/sanitizer_racecheck_sync.log 2>&1; echo "racecheck sync rc=$?"; tail -2 gpurun_out/sanitizer_racecheck_sync.log
python tools/gemm_dct_ab.py > gpurun_out/gemm_dct_ab.jsonl 2>&1; cat gpurun_out/gemm_dct_ab.jsonl
ncu --metrics sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active,gpu__time_duration.sum --clock-control none \
   -k regex:"gemm|Kernel|sm100|cutlass" -c 6 python tools/gemm_dct_ab.py > gpurun_out/gemm_dct_ncu.txt 2>&1; grep -E "tensor|duration|Kernel|void" gpurun_out/gemm_dct_ncu.txt | head -30
