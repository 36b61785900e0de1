# split WA launch around the field transforms (DP_WA_SPLIT = % of chunks beside the map) x field path
mkdir -p gpurun_out
echo "== parity split"; DP_WA_SPLIT=50 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_gp.py -x -q -k "eval or gp or initial or wl_grad" 2>&1 | tail -2
echo "== parity default"; timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "fields or shard or transforms" 2>&1 | tail -2
bash tools/ab_quick.sh DP_FFT=0 "DP_FFT=0 DP_WA_SPLIT=40" "DP_FFT=0 DP_WA_SPLIT=55" "DP_FFT=0 DP_WA_SPLIT=70" "DP_FFT=1 DP_WA_SPLIT=40" "DP_FFT=1 DP_WA_SPLIT=55" "DP_FFT=1 DP_WA_SPLIT=70" "DP_FFT=2 DP_WA_SPLIT=55"
