DP_PDL=1 timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_gp.py tests/test_gpu_det.py -x -q -k "not slow and not adaptec1" > gpurun_out/t_pdl.log 2>&1; tail -2 gpurun_out/t_pdl.log
bash tools/ab_quick.sh "DP_PDL=1" "DP_PDL=0" "DP_PDL=1" "DP_PDL=0" > gpurun_out/ab_pdl.txt 2>&1
