python -c "import sys; sys.path.insert(0,'.'); from paper_conf_dac_lindlrkp19_b200.build import build; build()"
python tools/gemm_dct_ab.py > gpurun_out/gemm_dct_ab.jsonl 2>&1; cat gpurun_out/gemm_dct_ab.jsonl
ncu --metrics sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_tensor.sum,gpu__time_duration.sum --clock-control none \
   -k regex:"nvjet|gemm|xmma|sm100|cutlass" -s 200 -c 6 python tools/gemm_dct_ab.py > gpurun_out/gemm_dct_ncu.txt 2>&1
grep -E "nvjet|gemm|xmma|sm100|tensor|duration" gpurun_out/gemm_dct_ncu.txt | head -30
bash tools/ab_quick.sh "DP_X=0" "DP_FUSED_T2=1" "DP_T1_TMA=1" "DP_X=0" "DP_FUSED_T2=1"
