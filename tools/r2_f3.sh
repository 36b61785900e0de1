# radix-16 in-place CTA FFT field passes: parity (forced everywhere and default), fields alone, step A/B, ncu
mkdir -p gpurun_out
echo "== parity DP_FFT=1"; DP_FFT=1 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "transforms or fields or eval or initial or sweep or shard or industrial" 2>&1 | tail -4
echo "== parity DP_FFT=2"; DP_FFT=2 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "transforms or fields or eval_tiny or initial" 2>&1 | tail -2
echo "== parity default"; timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "fields_sizes or industrial or shard" 2>&1 | tail -2
for f in 0 1 2; do echo "== chain DP_FFT=$f"; DP_FFT=$f python tools/chain_times.py bigblue4; done
bash tools/ab_quick.sh DP_FFT=0 DP_FFT=1 DP_FFT=2 DP_FFT=0 DP_FFT=1 DP_FFT=2
DP_FFT=1 ncu --set full --clock-control none --import-source on -k regex:"k_p[123]" --launch-skip 60 --launch-count 3 \
    -o gpurun_out/prof_f16b python tools/chain_times.py bigblue4 > gpurun_out/ncu_f16b.log 2>&1
