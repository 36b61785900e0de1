# fields at 1024^2 alone: chain stage times (warp FFT vs CTA FFT) and ncu --set full of both pass sets
mkdir -p gpurun_out
for f in 0 1; do echo "== DP_FFT=$f"; DP_FFT=$f python tools/chain_times.py bigblue4; done
DP_FFT=1 ncu --set full --clock-control none --import-source on -k regex:"k_p[123]" --launch-skip 60 --launch-count 3 \
    -o gpurun_out/prof_fcta python tools/chain_times.py bigblue4 > gpurun_out/ncu_fcta.log 2>&1
DP_FFT=0 ncu --set full --clock-control none --import-source on -k regex:"k_(row_dct|col_fwd|row_inv)" --launch-skip 80 --launch-count 4 \
    -o gpurun_out/prof_fwarp python tools/chain_times.py bigblue4 > gpurun_out/ncu_fwarp.log 2>&1
ls gpurun_out
